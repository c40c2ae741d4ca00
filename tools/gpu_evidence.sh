#!/bin/bash
# One gpurun call that refreshes every measured artifact under profiles/ (read back here with
# tools/ncu_summary.py, tools/configs_table.py, tools/model_fit.py):
#   bench line (default), the §8(d) config sweep, the V-cycle launch list, ncu --set full of the
#   level-0 two-sweep pass (sweep2_kernel<0>) and of the warp-stream variant (sweep2w_kernel<0>).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
timeout 1500 python tools/config_sweep.py --out gpurun_out/configs.json > gpurun_out/configs.log 2>&1; echo "sweep rc=$?"
ARGS="--steps 2 --warmup 1 --no-cpu-baseline --no-e2e"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 260 --csv \
   --log-file gpurun_out/launches.csv python bench.py $ARGS > gpurun_out/ncu_launch_run.log 2>&1; echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep2_kernel -s 2 -c 1 \
   -o gpurun_out/prof_sweep2 -f python bench.py $ARGS > gpurun_out/ncu_full_run.log 2>&1; echo "full rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep2w -s 2 -c 1 \
   -o gpurun_out/prof_sweep2w -f python bench.py $ARGS --tb 2 > gpurun_out/ncu_w.log 2>&1; echo "full w rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:coarse_cluster -s 1 -c 1 \
   -o gpurun_out/prof_coarse -f python bench.py $ARGS > gpurun_out/ncu_c.log 2>&1; echo "full coarse rc=$?"
tail -2 gpurun_out/smoke.log; cut -c1-400 gpurun_out/bench.json

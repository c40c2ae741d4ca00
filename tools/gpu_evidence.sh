#!/bin/bash
# One gpurun call that refreshes the measured artifacts under profiles/ (read back here with
# tools/ncu_summary.py, tools/configs_table.py, tools/model_fit.py):
#   bench line (default), the launch list of the bench command, ncu --set full of the level-0
#   pencil two-sweep pass (sweep2p_kernel<0>), optionally (CONFIGS=1) the §8(d) config sweep.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
ARGS="--steps 2 --warmup 1 --no-cpu-baseline --no-e2e"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 260 --csv \
   --log-file gpurun_out/launches.csv python bench.py $ARGS > gpurun_out/ncu_launch_run.log 2>&1; echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep2p_kernel -s 2 -c 1 \
   -o gpurun_out/prof_sweep2p -f python bench.py $ARGS > gpurun_out/ncu_full_run.log 2>&1; echo "full rc=$?"
if [ -n "$CONFIGS" ]; then
  timeout 1800 python tools/config_sweep.py --out gpurun_out/configs.json > gpurun_out/configs.log 2>&1; echo "sweep rc=$?"
fi
tail -2 gpurun_out/smoke.log; cut -c1-400 gpurun_out/bench.json

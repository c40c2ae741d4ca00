#!/bin/bash
# Final round-2 evidence in one gpurun call: build + smoke, the full GPU suite, the bench line, the
# launch lists of the default cycle and of the N4 variants (Fig 7 view of their level-0 kernels), one
# ncu --set full of the level-0 pencil pass (profiles/r02_sweep2p_full.md, ncu_sweep_summary.json).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/fin
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/fin/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/fin/smoke.log
if [ "${PYTEST:-1}" = "1" ]; then
  timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/fin/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/fin/pytest_gpu.log
fi
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/fin/bench.json 2> gpurun_out/fin/bench.err; echo "bench rc=$?"
A="--steps 2 --warmup 1 --no-cpu-baseline --no-e2e"
M="--metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv"
timeout 900 ncu $M -c 400 --log-file gpurun_out/fin/launches.csv python bench.py $A > /dev/null 2>&1; echo "launches rc=$?"
for v in "varcoef --var-coef" "brick4 --brick-edge 4" "dirichlet --bc 1" "paper --fusion 1 --tb 0" "ghostall_peer --ghost-all --transport peer"; do
  set -- $v
  tag=$1; shift
  timeout 900 ncu $M -c 800 --log-file gpurun_out/fin/launches_$tag.csv python bench.py $A "$@" > /dev/null 2>&1; echo "launches $tag rc=$?"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep2p_kernel -s 2 -c 1 \
   -o gpurun_out/fin/prof_pass -f python bench.py $A > gpurun_out/fin/ncu_full.log 2>&1; echo "full rc=$?"
if [ "${CONFIGS:-0}" = "1" ]; then
  timeout 1800 python tools/config_sweep.py --out gpurun_out/fin/configs.json > gpurun_out/fin/configs.log 2>&1; echo "configs rc=$?"
fi

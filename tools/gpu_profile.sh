#!/bin/bash
# ncu evidence for the bench workload: (1) launch list with per-launch device time,
# (2) one `ncu --set full` capture of the level-0 sweep kernel.  Never a bench number.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
ARGS="--steps 2 --warmup 1 --no-cpu-baseline --no-e2e ${BENCH_ARGS}"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c ${NCU_COUNT:-260} --csv \
   --log-file gpurun_out/launches.csv python bench.py $ARGS > gpurun_out/ncu_launch_run.log 2>&1
echo "launch list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-sweep_kernel} \
   -s ${NCU_SKIP:-40} -c ${NCU_C:-1} -o gpurun_out/prof_sweep -f python bench.py $ARGS > gpurun_out/ncu_full_run.log 2>&1
echo "full rc=$?"
ls -la gpurun_out/

#!/bin/bash
# One gpurun call (round 2 iteration): build, smoke, GPU tests, bench (default and A/B variants),
# the launch list and one ncu --set full capture of the level-0 pass kernel.
#   BENCH_AB="--tb 3;--tb 1 --bottom-mode 4"   extra bench variants (';'-separated), short runs
#   NCU_KERNEL=sweep2q_kernel                   regex of the kernel to capture (empty: skip)
#   PYTEST_ARGS="-x -q"                         GPU test selection (PYTEST=0: skip)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" | tee -a gpurun_out/smoke.log
tail -1 gpurun_out/smoke.log
if [ "${PYTEST:-1}" = "1" ]; then
  timeout ${PYTEST_TIMEOUT:-1500} python -m pytest tests -m gpu ${PYTEST_ARGS:--q --maxfail=10} > gpurun_out/pytest_gpu.log 2>&1
  echo "pytest rc=$?"; tail -12 gpurun_out/pytest_gpu.log
fi
timeout 900 python bench.py ${BENCH_ARGS:---steps 20 --warmup 5} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
python - <<'PY'
import json
d = json.loads(open("gpurun_out/bench.json").read().strip().splitlines()[-1])
print("value %.4g ms %.3f roof %.3f achieved %.0f launch_ms %.4f launches %s" % (d["value"], d["ms_per_step"], d["roofline"]["frac"], d["roofline"]["achieved"], d["roofline"]["launch_ms"], d["launches_per_step"]))
for l in d["levels"]: print(" ", l)
PY
IFS=';' read -ra AB <<< "${BENCH_AB:-}"
i=0
for v in "${AB[@]}"; do
  i=$((i+1))
  timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e $v > gpurun_out/bench_ab$i.json 2> gpurun_out/bench_ab$i.err
  python - "$i" "$v" <<'PY'
import json, sys
try:
    d = json.loads(open(f"gpurun_out/bench_ab{sys.argv[1]}.json").read().strip().splitlines()[-1])
    print("AB[%s] %s: ms %.3f roof %.3f launch_ms %.4f" % (sys.argv[1], sys.argv[2], d["ms_per_step"], d["roofline"]["frac"], d["roofline"]["launch_ms"]))
    for l in d["levels"]: print("   ", l)
except Exception as e:
    print("AB", sys.argv[1], sys.argv[2], "failed", e)
PY
done
ARGS="--steps 2 --warmup 1 --no-cpu-baseline --no-e2e"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 400 --csv \
   --log-file gpurun_out/launches.csv python bench.py $ARGS > gpurun_out/ncu_launch_run.log 2>&1; echo "launches rc=$?"
if [ -n "${NCU_KERNEL:-}" ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${NCU_KERNEL} -s 2 -c 1 \
     -o gpurun_out/prof_pass -f python bench.py $ARGS > gpurun_out/ncu_full_run.log 2>&1; echo "full rc=$?"
fi

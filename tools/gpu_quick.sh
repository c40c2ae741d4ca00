#!/bin/bash
# Scratch GPU check used while developing a kernel: build, selected tests, bench A/B, launch list.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pt3.log 2>&1; echo "rc=$?" >> gpurun_out/pt3.log
tail -5 gpurun_out/pt3.log
for tb in ${TBS:-1 3}; do
  timeout 600 python bench.py --steps 20 --warmup 5 --tb $tb --no-cpu-baseline --no-e2e > gpurun_out/bench_tb$tb.json 2> gpurun_out/bench_tb$tb.err
  python -c "import json;d=json.load(open('gpurun_out/bench_tb$tb.json'));print('tb',$tb,d['ms_per_step'],d['value']/1e9,d['roofline']['launch_ms'],d['roofline']['frac'])"
done
ARGS="--steps 2 --warmup 1 --no-cpu-baseline --no-e2e --tb ${NCU_TB:-3}"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 140 --csv \
   --log-file gpurun_out/launches_q.csv python bench.py $ARGS > gpurun_out/ncu_q.log 2>&1; echo "launches rc=$?"

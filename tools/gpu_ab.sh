#!/bin/bash
# Scratch A/B on one GPU: build, GPU tests (optional), bench lines for each argument set in AB
# (separated by ';'), e.g.  AB="--no-pdl;" bash tools/gpu_ab.sh
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
if [ -z "$NOTEST" ]; then
  timeout 1200 python -m pytest tests -m gpu -q -x ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pt_ab.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pt_ab.log
  tail -3 gpurun_out/pt_ab.log
fi
IFS=";" read -ra SETS <<< "${AB:-}"; [ ${#SETS[@]} -eq 0 ] && SETS=("")
i=0
for rep in ${REPS:-1 2}; do
for args in "${SETS[@]}"; do
  timeout 600 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e $args > gpurun_out/ab_$i.json 2> gpurun_out/ab_$i.err
  python - "$i" "$args" <<'PY'
import json, sys
i, args = sys.argv[1], sys.argv[2]
try:
    d = json.load(open(f"gpurun_out/ab_{i}.json"))
    lv = " ".join(f"L{l['level']}:" + "+".join(f"{k}={v:.4f}" for k, v in l['ms'].items()) for l in d['levels'])
    print(f"[{args}] ms={d['ms_per_step']:.4f} GDOF/s={d['value']/1e9:.3f} pass={d['roofline']['launch_ms']:.4f} frac={d['roofline']['frac']:.4f} clk={d['clocks']['sm_mhz']} | {lv}")
except Exception as e:
    print(f"[{args}] failed: {e}"); print(open(f"gpurun_out/ab_{i}.err").read()[-2000:])
PY
  i=$((i+1))
done
done

#!/bin/bash
# Self-exchange (ghost shell on every axis) V-cycles on one GPU over local copies and NCCL, CA periods
# 2 / 4 / 8, against the no-ghost cycle: the bench lines (with the exchange block) under gpurun_out/xs/.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/xs
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "exchange_plan or self_exchange or peer_transport" 2>&1 | tail -2
run() { timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e "$@"; }
run > gpurun_out/xs/base.json 2>/dev/null
for t in local peer nccl; do for k in 0 8 4 2; do
  run --ghost-all --transport $t --ca-period $k > gpurun_out/xs/ga_${t}_k$k.json 2> gpurun_out/xs/ga_${t}_k$k.err
done; done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/xs/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "failed", e); continue
    ex = d.get("exchange", {})
    lv = " ".join("L%d:%dx%.3fms(%.0fGB/s)" % (e["level"], e["exchanges_per_cycle"], e["ms_per_exchange"], e["gbs"] or 0)
                  for e in ex.get("levels", []))
    print("%-40s ms %.3f  levels %s" % (f.split("/")[-1], d["ms_per_step"], [round(sum(l["ms"].values()), 3) for l in d["levels"]]))
    if lv: print("    ", lv, "fit", ex.get("fit"))
PY

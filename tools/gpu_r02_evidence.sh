#!/bin/bash
# Round-2 evidence in one gpurun call: build + smoke, the default bench line, the variant bench lines
# (Dirichlet, variable coefficients, 4^3 bricks, self-exchanged ghost shells over local / peer / NCCL
# with their exchange fits), the ncu launch lists of the default cycle and of the paper's kernel set
# (fusion 1, one sweep per pass: the Fig 7 view of P:L296-302), one ncu --set full of the norm kernel.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/ev
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/ev/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/ev/smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/ev/bench.json 2> gpurun_out/ev/bench.err; echo "bench rc=$?"
run() { out=$1; shift; timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e "$@" > gpurun_out/ev/$out.json 2> gpurun_out/ev/$out.err; echo "$out rc=$?"; }
run dirichlet --bc 1
run neumann --bc 2
run varcoef --var-coef
run brick4 --brick-edge 4
run ga_local --ghost-all --transport local
run ga_peer --ghost-all --transport peer
run ga_nccl --ghost-all --transport nccl
run ga_nccl_k8 --ghost-all --transport nccl --ca-period 8
run paper_set --fusion 1 --tb 0
A="--steps 2 --warmup 1 --no-cpu-baseline --no-e2e"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 400 --csv \
   --log-file gpurun_out/ev/launches.csv python bench.py $A > /dev/null 2>&1; echo "launches rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 400 --csv \
   --log-file gpurun_out/ev/launches_paper.csv python bench.py $A --fusion 1 --tb 0 > /dev/null 2>&1; echo "paper launches rc=$?"
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ev/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "failed", e); continue
    ex = d.get("exchange", {})
    print("%-28s %.4g DOF/s  %.3f ms  roof %.3f  launches %s" % (f.split("/")[-1], d["value"], d["ms_per_step"],
          d.get("roofline", {}).get("frac", 0), d.get("gpu_launches")))
    print("    levels", [(l["level"], round(sum(l["ms"].values()), 3)) for l in d.get("levels", [])])
    if ex.get("levels"):
        print("    exch", [(e["level"], e["exchanges_per_cycle"], round(e["ms_per_exchange"], 4)) for e in ex["levels"]], "fit", ex.get("fit"))
PY

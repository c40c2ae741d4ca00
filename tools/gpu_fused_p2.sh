#!/bin/bash
# Full GPU suite, then period 2 on fused levels (default) vs period 8 above level 0 (MG_FUSED_P8=1) vs the
# separate exchange (MG_NO_FUSED_EXCH=1), self-exchanged ghost shell on every axis; then the rehearsal.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pt_p2.log 2>&1; echo "pytest rc=$?"; grep -E "^E  |FAILED|passed|failed" gpurun_out/pt_p2.log | tail -8
run() { timeout 300 env $1 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e ${@:2} 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('%-52s %.4f ms  levels %s' % (sys.argv[1], d['ms_per_step'], [round(sum(l['ms'].values()),3) for l in d['levels']]))" "$*"; }
for rep in 1 2; do
  run X=1
  run X=1 --ghost-all --transport local
  run MG_FUSED_P8=1 --ghost-all --transport local
  run X=1 --ghost-all --transport peer
  run MG_FUSED_P8=1 --ghost-all --transport peer
  run MG_NO_FUSED_EXCH=1 --ghost-all --transport peer
done
timeout 900 python tools/loopback_scaling.py > gpurun_out/loopback_p2.md 2> gpurun_out/loopback_p2.err; grep "^| 2x\|Single\|^\* 2x" gpurun_out/loopback_p2.md

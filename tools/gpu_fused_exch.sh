#!/bin/bash
# Exchange fused into the pencil passes (SW_PEER): GPU tests, then the self-exchanged ghost shell on
# every axis (the 2x2x2 halo pattern on one GPU) with the fused passes vs the separate exchange
# kernel (MG_NO_FUSED_EXCH=1), against the cycle without a ghost shell; then the loopback rehearsal.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
if [ -z "$NOTEST" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -x ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pt_fx.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pt_fx.log
  tail -15 gpurun_out/pt_fx.log
fi
run() { timeout 300 env $1 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e ${@:2} 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('%-52s %.4f ms  levels %s' % (sys.argv[1], d['ms_per_step'], [round(sum(l['ms'].values()),3) for l in d['levels']]))" "$*"; }
for rep in 1 2; do
  run X=1
  run X=1 --ghost-all --transport local
  run MG_NO_FUSED_EXCH=1 --ghost-all --transport local
  run X=1 --ghost-all --transport peer
  run MG_NO_FUSED_EXCH=1 --ghost-all --transport peer
done
timeout 600 python tools/loopback_scaling.py > gpurun_out/loopback_fx.md 2> gpurun_out/loopback_fx.err; grep "^| 2x\|Single" gpurun_out/loopback_fx.md
MG_NO_FUSED_EXCH=1 timeout 600 python tools/loopback_scaling.py > gpurun_out/loopback_nofx.md 2>&1; grep "^| 2x\|Single" gpurun_out/loopback_nofx.md

#!/bin/bash
# Cluster-resident bottom (bottom_cluster.cu) A/B: GPU tests, then the bottom of a 64-brick coarsest
# level (one rank: 512^3 L = 5, 256^3 L = 4) and the loopback 2x2x2 rehearsal (replicated 64-brick
# bottom) with the cluster kernel vs without (MG_NO_CLUSTER_BOTTOM=1: per-sweep launches / coarse.cu).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
if [ -z "$NOTEST" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -x ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pt_cb.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pt_cb.log
  tail -3 gpurun_out/pt_cb.log
fi
run() { timeout 300 env $1 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e ${@:2} 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('%-44s %.4f ms  levels %s' % (sys.argv[1], d['ms_per_step'], [(l['level'], l['ms']) for l in d['levels'][-2:]]))" "$*"; }
for rep in 1 2; do
  run X=1 --levels 5
  run MG_NO_CLUSTER_BOTTOM=1 --levels 5
  run X=1 --n 256 --levels 4
  run MG_NO_CLUSTER_BOTTOM=1 --n 256 --levels 4
done
timeout 600 python tools/loopback_scaling.py > gpurun_out/loopback_cb.md 2> gpurun_out/loopback_cb.err; tail -12 gpurun_out/loopback_cb.md
MG_NO_CLUSTER_BOTTOM=1 timeout 600 python tools/loopback_scaling.py > gpurun_out/loopback_nocb.md 2>&1; tail -12 gpurun_out/loopback_nocb.md

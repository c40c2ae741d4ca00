#!/bin/bash
# Cluster bottom: bricks per CTA (16-CTA clusters by default) and the cluster for the 8-brick bottom
# (MG_BC_SMALL=1) -- parity subsets under each setting, then interleaved bench A/B.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
K="bottom or bc_vcycle or loopback or replicated or smoke or full_size_512_vcycle"
for envs in X=1 MG_BC_BPC=8 MG_BC_SMALL=1 "MG_BC_SMALL=1 MG_BC_BPC=2"; do
  env $envs timeout 900 python -m pytest tests -m gpu -q -x -k "$K" > gpurun_out/pt_cb2.log 2>&1; echo "[$envs] pytest rc=$? $(tail -1 gpurun_out/pt_cb2.log)"
done
run() { timeout 300 env $1 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e ${@:2} 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('%-44s %.4f ms  levels %s' % (sys.argv[1], d['ms_per_step'], [(l['level'], l['ms']) for l in d['levels'][-1:]]))" "$*"; }
for rep in 1 2; do
  run X=1 --n 256 --levels 4
  run MG_BC_BPC=8 --n 256 --levels 4
  run MG_BC_BPC=2 --n 256 --levels 4
  run X=1
  run MG_BC_SMALL=1
  run "MG_BC_SMALL=1 MG_BC_BPC=2"
  run "MG_BC_SMALL=1 MG_BC_BPC=4"
done
timeout 600 python tools/loopback_scaling.py > gpurun_out/loopback_cb.md 2> gpurun_out/loopback_cb.err; grep "^| 2x" gpurun_out/loopback_cb.md
MG_BC_SMALL=1 timeout 600 python tools/loopback_scaling.py > gpurun_out/loopback_cbs.md 2>&1; grep "^| 2x\|Single" gpurun_out/loopback_cbs.md

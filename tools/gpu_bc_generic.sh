#!/bin/bash
# Cluster bottom with generic neighbour addresses: parity subset, the 64-brick bottom in the bench, ncu.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/fin
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q -x -k "bottom or bc_vcycle or loopback or replicated or peer_transport" > gpurun_out/pt_bc.log 2>&1; echo "pytest rc=$? $(tail -1 gpurun_out/pt_bc.log)"
for rep in 1 2 3; do
  timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e --n 256 --levels 4 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('%.4f ms' % d['ms_per_step'], d['levels'][-1])"
done
BC=1 bash tools/gpu_ncu_new.sh > /dev/null 2>&1; ls gpurun_out/fin/prof_bc.ncu-rep

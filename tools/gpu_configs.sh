#!/bin/bash
# One gpurun call: the §8(d) config sweep (tools/config_sweep.py) and one ncu capture of the
# warp-stream two-sweep kernel (temporal_blocking = 2).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1500 python tools/config_sweep.py --out gpurun_out/configs.json ${SWEEP_ARGS} > gpurun_out/configs.log 2>&1; echo "sweep rc=$?"
tail -3 gpurun_out/configs.log
echo "ncu rc=$?"

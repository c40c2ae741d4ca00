#!/bin/bash
# Scratch check of the warp-stream two-sweep kernel (temporal_blocking = 2).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 120 python -m pytest tests -m gpu -q -x -k "two_sweep_pass_per_op and 2-" > gpurun_out/t0.log 2>&1; echo "t0 rc=$?"; tail -30 gpurun_out/t0.log
timeout 900 python -m pytest tests -m gpu -q -k "tb or two_sweep" > gpurun_out/t1.log 2>&1; echo "t1 rc=$?"; tail -30 gpurun_out/t1.log
timeout 300 python tools/ab_vcycle.py --n 512 --levels 6 --variants tb=1 tb=2 2>&1 | tail -30

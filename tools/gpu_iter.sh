#!/bin/bash
# Kernel iteration on one GPU: build, GPU tests, bench (REPS times), ncu --set full of the level-0 pencil pass.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q -x ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pt_iter.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pt_iter.log
tail -3 gpurun_out/pt_iter.log
NOTEST=1 AB="${AB:-}" REPS="${REPS:-1 2}" bash tools/gpu_ab.sh | grep -v "^\[gpurun"
if [ -z "$NONCU" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sweep2p_kernel -s 2 -c 1 \
   -o gpurun_out/prof_iter -f python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_iter.log 2>&1; echo "ncu rc=$?"
fi

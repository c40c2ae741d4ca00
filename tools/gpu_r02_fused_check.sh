#!/bin/bash
# New-path checks: the fused-exchange / cluster-bottom tests (incl. 4- and 8-process peer runs with the
# handshake kernel).  (compute-sanitizer is closed on this pool.)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q -k "${PYTEST_K:-fused or peer_transport_multiprocess}" > gpurun_out/pt_new.log 2>&1
echo "pytest rc=$?"; grep -E "^E  |FAILED|passed|failed" gpurun_out/pt_new.log | tail -12

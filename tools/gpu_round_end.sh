#!/bin/bash
# End-of-round evidence in one gpurun call: the final evidence set (smoke, full GPU suite, bench line,
# launch lists, ncu of the pencil pass, config sweep) and the self-exchange transport sweep.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
CONFIGS=1 bash tools/gpu_final_evidence.sh
bash tools/gpu_exchange_sweep.sh > gpurun_out/fin/exchange_sweep.txt 2>&1; echo "exchange sweep rc=$?"
tail -40 gpurun_out/fin/exchange_sweep.txt

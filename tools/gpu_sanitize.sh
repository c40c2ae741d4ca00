#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over small V-cycles: the
# persistent TMA / mbarrier kernels (pencil passes, column streams, one-brick two-sweep streams),
# the one-brick sweeps, the resident bottom, the copy kernels of a self-exchanged ghost shell.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/sanitize
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck; do
  IFS=';' read -ra LIST <<< "${CFGS:-64 4 0 3 0;128 5 0 3 0;64 3 2 3 0;128 4 2 3 0;64 3 2 1 0;64 3 2 0 0;64 3 0 3 1}"
  for cfg in "${LIST[@]}"; do
    tag=$(echo $tool $cfg | tr ' ' '_')
    timeout 900 $CS --tool $tool --print-limit 20 python tools/sanitize_run.py $cfg \
       > gpurun_out/sanitize/$tag.log 2>&1
    echo "$tool [$cfg] rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|bitwise' gpurun_out/sanitize/$tag.log | tr '\n' ' ')"
  done
done | tee gpurun_out/sanitize/summary.txt

#!/bin/bash
# A/B of the interior / surface split of single-sweep levels (params overlap, bench --no-overlap) with a
# self-exchanged ghost shell on every axis (512^3, peer kernel and local copies; pencil split off).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 env $1 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e ${@:2} 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('%-58s %.3f ms  levels %s' % (sys.argv[1], d['ms_per_step'], [round(sum(l['ms'].values()),3) for l in d['levels']]))" "$*"; }
for rep in 1 2 3; do
  for t in peer local; do
    run MG_PENCIL_OVERLAP=0 --ghost-all --transport $t
    run MG_PENCIL_OVERLAP=0 --ghost-all --transport $t --no-overlap
  done
done

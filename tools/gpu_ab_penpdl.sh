#!/bin/bash
# Pencil passes launched with PDL on levels >= l0 (MG_PEN_PDL=l0) vs plain launches (default), interleaved.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 env $1 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e ${@:2} 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('%-30s %.4f ms  levels %s' % (sys.argv[1], d['ms_per_step'], [round(sum(l['ms'].values()),4) for l in d['levels']]))" "$*"; }
for rep in 1 2 3; do
  run X=1
  run MG_PEN_PDL=1
  run MG_PEN_PDL=2
  run MG_PEN_PDL=0
  run X=1 --n 256 --levels 5
  run MG_PEN_PDL=1 --n 256 --levels 5
done

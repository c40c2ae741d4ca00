#!/bin/bash
# Pencil CTAs per launch (MG_PEN_CTAS) -- for the per-level view: does level 1 / 2 prefer fewer CTAs?
cd "${GRAFT_REPO_ROOT:-/root/repo}"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 env $1 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e ${@:2} 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('%-30s %.4f ms  levels %s' % (sys.argv[1], d['ms_per_step'], [round(sum(l['ms'].values()),4) for l in d['levels']]))" "$*"; }
for rep in 1 2; do
  for c in 888 740 592 444 296; do run MG_PEN_CTAS=$c; done
done

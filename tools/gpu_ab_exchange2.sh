#!/bin/bash
# A/B of the auto CA period per level with depth-limited exchanges (512^3, self-exchanged ghost shell on
# every axis): period 2 on levels < MG_CA2_LEVELS (default 1), 8 below; local copies and peer kernel.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 env $1 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e ${@:2} 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); x=d.get('exchange',{})
print('%-50s %.3f ms  levels %s  exch %s' % (sys.argv[1], d['ms_per_step'], [round(sum(l['ms'].values()),3) for l in d['levels']],
      [(e.get('level'), e.get('exchanges_per_cycle'), round(e.get('ms_per_exchange',0),4)) for e in x.get('levels',[])]))" "$*"; }
for rep in 1 2; do
  run X=1
  for t in local peer; do
    for n in 1 2 3 4 5; do run MG_CA2_LEVELS=$n --ghost-all --transport $t; done
  done
done

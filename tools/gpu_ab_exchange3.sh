#!/bin/bash
# Per-level CA periods with depth-limited exchanges (MG_CA_AUTO="k0,k1,..."; 512^3, self-exchanged ghost
# shell on every axis, peer kernel and local copies; interleaved).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 env $1 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e ${@:2} 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('%-46s %.3f ms  levels %s' % (sys.argv[1], d['ms_per_step'], [round(sum(l['ms'].values()),3) for l in d['levels']]))" "$*"; }
for rep in 1 2; do
  for t in peer local; do
    for k in "2,8,8,8,8" "2,4,8,8,8" "2,4,4,8,8" "2,4,4,4,8" "4,4,8,8,8"; do run MG_CA_AUTO=$k --ghost-all --transport $t; done
  done
done

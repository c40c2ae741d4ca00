#!/bin/bash
# A/B of the pencil-pass exchange overlap (MG_PENCIL_OVERLAP: part 1 = units that read no ghost brick
# swept while the exchange runs, part 2 after it) on one GPU, 512^3 with a self-exchanged ghost shell
# on every axis over the peer kernel and local copies (interleaved).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 env $1 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e ${@:2} 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('%-52s %.3f ms  levels %s' % (sys.argv[1], d['ms_per_step'], [round(sum(l['ms'].values()),3) for l in d['levels']]))" "$*"; }
for rep in 1 2 3; do
  for t in peer local; do
    for o in 0 1; do run MG_PENCIL_OVERLAP=$o --ghost-all --transport $t; done
  done
done

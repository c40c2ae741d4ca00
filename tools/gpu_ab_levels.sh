#!/bin/bash
# A/B of coarse-level choices (measurement switches, 512^3 bench, interleaved): two-sweep pencil passes
# from 512 / 64 bricks on (MG_PAIR_MIN_BRICKS) and fewer pencil CTAs (MG_PEN_CTAS).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 env "$@" python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('%-28s %.3f ms  levels %s' % (sys.argv[1], d['ms_per_step'], [round(sum(l['ms'].values()),3) for l in d['levels']]))" "$*"; }
for rep in 1 2; do
  run X=default
  run MG_PAIR_MIN_BRICKS=512
  run MG_PAIR_MIN_BRICKS=64
  run MG_PEN_CTAS=740
  run MG_PEN_CTAS=592
done

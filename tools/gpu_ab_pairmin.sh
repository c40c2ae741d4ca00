#!/bin/bash
# Two-sweep passes on the small levels too (MG_PAIR_MIN_BRICKS=64 / 512: levels 3-4) vs the default
# (>= 4096 bricks), interleaved, 512^3 L = 6 and 256^3 L = 5.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 env $1 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e ${@:2} 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('%-44s %.4f ms  levels %s' % (sys.argv[1], d['ms_per_step'], [round(sum(l['ms'].values()),3) for l in d['levels']]))" "$*"; }
for rep in 1 2 3; do
  run X=1
  run MG_PAIR_MIN_BRICKS=512
  run MG_PAIR_MIN_BRICKS=64
  run X=1 --n 256 --levels 5
  run MG_PAIR_MIN_BRICKS=64 --n 256 --levels 5
done

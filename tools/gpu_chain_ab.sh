#!/bin/bash
# Chained pencil passes (sweep2p.cu CHAIN): parity first, then the bench A/B against one launch per
# pass (MG_PEN_CHAIN=0), interleaved.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "config2 or full_size_512_vcycle or vcycle_config1 or smoke or solve_matches or temporal_blocking_on_off" 2>&1 | tail -2
run() { timeout 300 env "$@" python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('%-22s %.3f ms  roof %.3f (pass %.4f ms)  levels %s' % (sys.argv[1], d['ms_per_step'], d['roofline']['frac'], d['roofline']['launch_ms'], [round(sum(l['ms'].values()),3) for l in d['levels']]))" "$*"; }
for rep in 1 2 3; do
  run X=chain
  run MG_PEN_CHAIN=0
done

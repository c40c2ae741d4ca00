#!/bin/bash
# A/B of the depth-limited ghost exchange (512^3, self-exchanged ghost shell on every axis = the halo
# pattern of a 2x2x2 decomposition on one GPU; interleaved): copy only the ghost cells within the
# exchange period (default) vs whole bricks (MG_EXCH_WHOLE=1), local copies and the peer kernel,
# against the cycle without a ghost shell.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 env $1 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e ${@:2} 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); x=d.get('exchange',{})
print('%-58s %.3f ms  levels %s  exch %s' % (sys.argv[1], d['ms_per_step'], [round(sum(l['ms'].values()),3) for l in d['levels']],
      [(e.get('level'), e.get('exchanges_per_cycle'), round(e.get('ms_per_exchange',0),4), e.get('bytes_per_exchange')) for e in x.get('levels',[])]))" "$*"; }
for rep in 1 2; do
  run X=1
  run X=1 --ghost-all --transport local
  run MG_EXCH_WHOLE=1 --ghost-all --transport local
  run X=1 --ghost-all --transport peer
  run MG_EXCH_WHOLE=1 --ghost-all --transport peer
  run X=1 --ghost-all --transport peer --ca-period 8
done

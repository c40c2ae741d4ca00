#!/bin/bash
# A/B of the one-brick sweep kernel: 128 threads (four cells each, default for ranges >= 4096 bricks) vs
# 256 threads everywhere (MG_SWEEP_NT256=1), on the cycles that use it at level 0 (variable
# coefficients, the paper's kernel set) and the default cycle (coarse levels only).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_variants.py tests/test_gpu_parity.py -q -x -k "var_coef or fusion or per_op or config1 or full_size_512_vcycle or norm" 2>&1 | tail -2
run() { e=$1; shift; timeout 300 env $e python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e "$@" 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('%-40s %.3f ms  levels %s' % (sys.argv[1], d['ms_per_step'], [round(sum(l['ms'].values()),3) for l in d['levels']]))" "$e $*"; }
for rep in 1 2; do
  run X=1 --var-coef
  run MG_SWEEP_NT256=1 --var-coef
  run X=1 --fusion 1 --tb 0
  run MG_SWEEP_NT256=1 --fusion 1 --tb 0
  run X=1
  run MG_SWEEP_NT256=1
done

#!/bin/bash
# Rehearsal of the multi-rank bench path on a one-GPU box (MG_BENCH_SHARED_GPU=1: ranks share the GPU,
# gloo for torch.distributed, ghosts over peer memory): the JSON line must come out of rank 0 with the
# exchange block; the peer transport for a 2x2x2 decomposition (8 processes) and a Dirichlet one
# against the oracle; the reference arm under torchrun.  Not measurements: the ranks' contexts time-share
# the GPU, and a rank's flag-waiting exchange kernel holds it while its peer's work waits for the slice.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
TR="python -m torch.distributed.run --nnodes=1 --master-addr 127.0.0.1"
for np_n in "2 256 6" "4 128 5" "8 128 5"; do
  set -- $np_n
  MG_BENCH_SHARED_GPU=1 timeout 900 $TR --nproc-per-node $1 --master-port $((29500 + $1)) bench.py --gpus $1 --size $2 \
     --levels $3 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/reh_$1.json 2> gpurun_out/reh_$1.err
  echo "N=$1 rc=$? $(tail -c 400 gpurun_out/reh_$1.json | head -c 300)"
done
python - <<'PY'
import json
for n in (2, 4, 8):
    try:
        d = json.loads(open(f"gpurun_out/reh_{n}.json").read().strip().splitlines()[-1])
        ex = d.get("exchange", {})
        print(n, d["n_gpus"], d["config"]["proc_grid"], "%.3f ms" % d["ms_per_step"], "e2e", d["e2e"]["value"] > 0,
              "exch levels", [(e["level"], e["exchanges_per_cycle"]) for e in ex.get("levels", [])], ex.get("transport"))
    except Exception as e:
        print(n, "failed", e)
PY
for cfg in "16 16 16 2 2 2 2 2 0" "32 32 32 2 1 1 3 2 0 1" "16 16 32 2 2 2 2 2 1 2"; do
  set -- $cfg
  timeout 900 $TR --nproc-per-node $(($4 * $5 * $6)) --master-port 29611 tools/peer_check.py $cfg 2>&1 | grep -E "peer_check|Error|error" | head -3
done
timeout 900 $TR --nproc-per-node 2 --master-port 29622 bench.py --impl reference --gpus 2 --steps 1 --warmup 0 2>/dev/null | tail -1 | head -c 300; echo

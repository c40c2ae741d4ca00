"""Multi-process check of the peer-memory (CUDA IPC) transport, one process per rank.

torchrun --nproc-per-node P --master-addr 127.0.0.1 --master-port PORT tools/peer_check.py NX NY NZ PX PY PZ L [NCYC] [GHOST] [BC]
NX..NZ: cells per rank; PX..PZ: process grid (P = PX*PY*PZ).  Every rank runs on cuda:(LOCAL_RANK % #GPUs)
(several ranks may share one GPU: CUDA IPC works between processes on the same device), sets its block
of a seeded global right-hand side, runs NCYC V-cycles and compares its x block and the global residual
norm with the CPU oracle on the undecomposed grid, bit for bit.  torch.distributed runs on gloo (only
the IPC blobs travel through it).  Rank 0 prints one line 'peer_check ok ...' or raises.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import mg_inputs  # noqa: E402
import oracle  # noqa: E402
from paper_conf_sc_antepara0jh24_b200 import mg  # noqa: E402
from paper_conf_sc_antepara0jh24_b200.solver import Multigrid  # noqa: E402


def main():
    a = [int(v) for v in sys.argv[1:]]
    nl, pg, L = tuple(a[0:3]), tuple(a[3:6]), a[6]
    ncyc = a[7] if len(a) > 7 else 2
    ghost = a[8] if len(a) > 8 else 0
    bc = a[9] if len(a) > 9 else 0  # non-periodic boundary (reading A22): mirrors on the outer ranks
    rank, world, local = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"]), int(os.environ["LOCAL_RANK"])
    assert world == pg[0] * pg[1] * pg[2]
    dist.init_process_group("gloo")
    dev = local % torch.cuda.device_count()
    torch.cuda.set_device(dev)
    gshape = (nl[2] * pg[2], nl[1] * pg[1], nl[0] * pg[0])
    b = mg_inputs.random_rhs(gshape, 7) if bc == 0 else mg_inputs.random_field(gshape, 7)
    m = Multigrid(nl, pg, L, rank=rank, world_size=world, device=dev, transport=mg.MG_TRANSPORT_PEER,
                  ghost_mode=ghost, bc=bc)
    m.set_rhs(torch.from_numpy(np.ascontiguousarray(mg_inputs.local_block(b, rank, pg))).cuda())
    m.set_solution(None)
    o = oracle.OracleMG(gshape, L, bc=bc)
    o.set_b(b)
    o.set_x(None)
    for c in range(ncyc):
        m.vcycle()
        o.vcycle()
        nr = m.residual_norm()
        want = mg_inputs.local_block(o.get_x(), rank, pg)
        x = m.get_solution().cpu().numpy()
        ok = np.array_equal(x, want) and nr == o.norm()
        flags = [None] * world
        dist.all_gather_object(flags, (ok, float(np.abs(x - want).max()), nr))
        if not all(f[0] for f in flags):
            raise SystemExit(f"peer_check FAILED cycle {c + 1} (rank, ok, max|dx|, norm): "
                             f"{[(r,) + f for r, f in enumerate(flags)]} oracle norm {o.norm()}")
    launches = m.launches_per_vcycle()
    fused = m.exchange_fused()  # exchanges fused into level pencil passes (SW_PEER + handshake kernel)
    m.close()
    if rank == 0:
        print(f"peer_check ok: {world} processes, proc grid {pg}, {nl} per rank, L={L}, ghost_mode={ghost}, bc={bc}, "
              f"{ncyc} V-cycles bitwise equal to the oracle (last norm {nr:.6e}, {launches} launches per cycle, "
              f"fused exchanges per level {fused})")
    dist.destroy_process_group()


if __name__ == "__main__":
    main()

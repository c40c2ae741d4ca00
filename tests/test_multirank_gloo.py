"""N>1 host path on CPU: world_size 2 and 4 processes over torch.distributed
(gloo, 127.0.0.1).  Each rank builds ITS OWN layout and exchange plan through
the C ABI (host-only queries), exchanges ghost bricks with real point-to-point
messages posted in plan order (the order NCCL relies on), runs the V-cycle in
the host brick interpreter, and the gathered solution must equal the
lexicographic oracle's bit for bit."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, n_local, pg, L, out_dir, replicated):
    import sys

    sys.path.insert(0, ROOT)
    import mg_inputs
    from paper_conf_sc_antepara0jh24_b200 import mg
    from tests import brick_interp as bi

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        p = mg.params(n_local, pg, num_levels=L)
        lay = mg.Layout(p, rank, world)
        levels = [bi.RankLevel(lay, l) for l in range(L)]

        def exchange(fields, lvls):
            f, Lv = fields[0], lvls[0]
            out = f.copy()
            reqs, bufs = [], []
            for peer, d, run, local, remote, count in Lv.recvs:
                if peer == rank:
                    out[local:local + count] = f[remote:remote + count]
                    continue
                buf = torch.empty(int(count) * 512, dtype=torch.float64)
                reqs.append(dist.irecv(buf, src=int(peer), tag=0))
                bufs.append((local, count, buf))
            for peer, d, run, local, remote, count in Lv.sends:
                if peer == rank:
                    continue
                t = torch.from_numpy(np.ascontiguousarray(f[local:local + count]).ravel())
                reqs.append(dist.isend(t, dst=int(peer), tag=0))
            for q in reqs:
                q.wait()
            for local, count, buf in bufs:
                out[local:local + count] = buf.numpy().reshape(int(count), 8, 8, 8)
            return [out]

        gshape = (n_local[2] * pg[2], n_local[1] * pg[1], n_local[0] * pg[0])
        b = mg_inputs.random_rhs(gshape, 11)
        h0 = mg_inputs.default_h0(gshape)
        xs = [[levels[l].zeros() for l in range(L)]]
        bs = [[None] * L]
        bs[0][0] = exchange([levels[0].to_bricks(mg_inputs.local_block(b, rank, pg))], [levels[0]])[0]
        rep = lay.repl()
        assert rep is not None  # decomposed coarsest level with a ghost shell, tiny global grid

        def gathered(b_own):  # the all-gather the library does with ncclAllGather, rank-major
            n_own = b_own.shape[0]
            parts = [torch.empty(n_own * 512, dtype=torch.float64) for _ in range(world)]
            dist.all_gather(parts, torch.from_numpy(np.ascontiguousarray(b_own).ravel()))
            return torch.cat(parts).numpy().reshape(world * n_own, 8, 8, 8)

        def bottom_fn(xs_, bs_, h):
            n_own = levels[L - 1].n_owned
            xs_[0][L - 1][:n_own] = bi.replicated_bottom(bs_[0][L - 1][:n_own], gathered, rep[0], rep[1], rep[2], h, 10)

        xs = bi.vcycle_ranks(xs, bs, [levels], L, h0, 2, 2, 10, exchange=exchange,
                             bottom_fn=bottom_fn if replicated else None)
        np.save(os.path.join(out_dir, f"x{rank}.npy"), levels[0].from_bricks(xs[0][0]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("replicated", [False, True])
@pytest.mark.parametrize("n_local,pg,L", [((16, 16, 16), (2, 1, 1), 2), ((16, 16, 16), (2, 2, 1), 2)])
def test_gloo_multirank_vcycle_bitwise(oracle_mod, tmp_path, n_local, pg, L, replicated):
    """Per-rank layouts and plans from the C ABI, real gloo point-to-point exchanges, the bottom either
    swept with ghost exchanges or replicated as the library does it (all-gather of the owned coarsest
    b over gloo, the library's gather / scatter maps and global adjacency): the oracle's bits."""
    import mg_inputs

    world = pg[0] * pg[1] * pg[2]
    mp.start_processes(_worker, args=(world, _free_port(), n_local, pg, L, str(tmp_path), replicated), nprocs=world,
                       join=True, start_method="spawn")
    gshape = (n_local[2] * pg[2], n_local[1] * pg[1], n_local[0] * pg[0])
    b = mg_inputs.random_rhs(gshape, 11)
    orc = oracle_mod.OracleMG(gshape, L, 2, 2, 10, mg_inputs.default_h0(gshape))
    orc.set_b(b)
    orc.set_x(None)
    orc.vcycle()
    want = orc.get_x()
    for r in range(world):
        got = np.load(os.path.join(tmp_path, f"x{r}.npy"))
        assert np.array_equal(got, mg_inputs.local_block(want, r, pg))

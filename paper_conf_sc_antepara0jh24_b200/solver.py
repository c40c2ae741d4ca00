"""Torch-facing wrappers over the C ABI (marshalling only).

``Multigrid`` owns one rank's context: it allocates the workspace as a torch
uint8 CUDA tensor, passes torch's stream, and (for world_size > 1) broadcasts
the NCCL unique id through ``torch.distributed``.  ``LoopbackGroup`` runs a
whole 3D decomposition inside one process on one GPU (ranks exchange ghost
bricks by device copies using the same exchange plan).  Every numerical step
happens in libmg_b200.so.
"""
from __future__ import annotations

import ctypes

import torch

from . import mg


def _ptr(t: torch.Tensor) -> int:
    return t.data_ptr()


class Multigrid:
    def __init__(self, n_local, proc_grid=(1, 1, 1), num_levels=6, pre=12, post=12, bottom=100, ca_period=None,
                 fusion=None, ghost_mode=mg.MG_GHOST_AUTO, transport=mg.MG_TRANSPORT_AUTO, use_graph=True,
                 bottom_mode=mg.MG_BOTTOM_AUTO, overlap=True, h0=0.0, rank=0, world_size=1, device=None,
                 stream: torch.cuda.Stream | None = None, sweep_kernel=0, temporal_blocking=3, smoother=0,
                 cheby_ratio=0, launch_pdl=0, bottom_solver=0, bc=0, var_coef=0, brick_edge=0):
        if not torch.cuda.is_available():
            raise RuntimeError("Multigrid needs a CUDA device (the library has no CPU fallback)")
        self.device = torch.device("cuda", torch.cuda.current_device() if device is None else int(device))
        torch.cuda.set_device(self.device)
        self.n_local = tuple(int(v) for v in n_local)  # (nx, ny, nz)
        self.num_levels = int(num_levels)
        self.rank, self.world_size = int(rank), int(world_size)
        self.p = mg.params(self.n_local, proc_grid, num_levels, pre, post, bottom, ca_period, fusion, ghost_mode,
                           transport, 1 if use_graph else 0, bottom_mode, 1 if overlap else 0, h0, sweep_kernel,
                           temporal_blocking, smoother, cheby_ratio, launch_pdl, bottom_solver, bc, var_coef,
                           brick_edge)
        self.ws_bytes = mg.mg_workspace_bytes(self.p, self.rank, self.world_size)
        self.ws = torch.empty(self.ws_bytes + 256, dtype=torch.uint8, device=self.device)
        base = _ptr(self.ws)
        self.ws_ptr = (base + 255) & ~255
        self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
        nccl_id = None
        self.transport = int(transport)
        peer = self.world_size > 1 and self.transport in (mg.MG_TRANSPORT_AUTO, mg.MG_TRANSPORT_PEER)
        if self.world_size > 1 and self.transport == mg.MG_TRANSPORT_NCCL:
            import torch.distributed as dist

            obj = [mg.mg_nccl_unique_id() if self.rank == 0 else None]
            dist.broadcast_object_list(obj, src=0)
            nccl_id = obj[0]
        self.ctx = mg.mg_setup(self.p, self.rank, self.world_size, nccl_id, self.device.index,
                               self.stream.cuda_stream, self.ws_ptr, self.ws_bytes)
        if peer:  # map every rank's workspace (CUDA IPC); blobs all-gathered in rank order
            import torch.distributed as dist

            blobs = [None] * self.world_size
            try:
                blob = mg.mg_peer_blob(self.ctx)
            except mg.MGError:
                blob = None
            dist.all_gather_object(blobs, blob)
            ok = all(b is not None for b in blobs)
            if ok:
                try:
                    mg.mg_peer_connect(self.ctx, b"".join(blobs))
                except mg.MGError:
                    ok = False
            oks = [None] * self.world_size
            dist.all_gather_object(oks, ok)
            if not all(oks):  # (e.g. no CUDA IPC between these devices): every rank falls back to NCCL
                mg.mg_destroy(self.ctx)
                self.ctx = None
                self.transport = mg.MG_TRANSPORT_NCCL
                self.p.transport = mg.MG_TRANSPORT_NCCL
                obj = [mg.mg_nccl_unique_id() if self.rank == 0 else None]
                dist.broadcast_object_list(obj, src=0)
                self.ctx = mg.mg_setup(self.p, self.rank, self.world_size, obj[0], self.device.index,
                                       self.stream.cuda_stream, self.ws_ptr, self.ws_bytes)

    @property
    def shape(self):  # numpy / torch order (nz, ny, nx)
        return (self.n_local[2], self.n_local[1], self.n_local[0])

    def close(self):
        if getattr(self, "ctx", None):
            mg.mg_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _check(self, t: torch.Tensor):
        assert t.dtype == torch.float64 and t.is_cuda and t.is_contiguous(), "fp64 contiguous CUDA tensor expected"
        assert tuple(t.shape) == self.shape, (tuple(t.shape), self.shape)

    def set_rhs(self, b: torch.Tensor):
        self._check(b)
        mg.mg_set_rhs(self.ctx, _ptr(b))

    def set_coefficients(self, c: torch.Tensor):
        """Cell coefficients c > 0 of the variable-coefficient variant (var_coef=1, reading A23)."""
        self._check(c)
        mg.mg_set_coefficients(self.ctx, _ptr(c))

    def set_rhs_host(self, b_host: torch.Tensor):
        assert b_host.dtype == torch.float64 and not b_host.is_cuda and b_host.is_contiguous()
        mg.mg_set_rhs_host(self.ctx, _ptr(b_host))

    def set_solution(self, x: torch.Tensor | None):
        if x is None:
            mg.mg_set_solution(self.ctx, None)
        else:
            self._check(x)
            mg.mg_set_solution(self.ctx, _ptr(x))

    def get_solution(self) -> torch.Tensor:
        out = torch.empty(self.shape, dtype=torch.float64, device=self.device)
        mg.mg_get_solution(self.ctx, _ptr(out))
        return out

    def get_solution_host(self, out: torch.Tensor | None = None) -> torch.Tensor:
        """x (local lexicographic) into a host fp64 tensor (pinned if allocated here); synchronises."""
        if out is None:
            out = torch.empty(self.shape, dtype=torch.float64, pin_memory=True)
        assert out.dtype == torch.float64 and not out.is_cuda and out.is_contiguous(), \
            "fp64 contiguous host tensor expected"
        assert tuple(out.shape) == self.shape, (tuple(out.shape), self.shape)
        mg.mg_get_solution_host(self.ctx, _ptr(out))
        return out

    def vcycle(self):
        mg.mg_vcycle(self.ctx)

    def residual_norm(self) -> float:
        return mg.mg_residual_norm(self.ctx)

    def residual_norm_async(self) -> None:
        mg.mg_residual_norm_async(self.ctx)

    def residual_norm_wait(self) -> float:
        return mg.mg_residual_norm_wait(self.ctx)

    def solve(self, tol=1e-10, max_cycles=20):
        return mg.mg_solve(self.ctx, tol, max_cycles)

    def level_shape(self, l):
        return tuple(s >> l for s in self.shape)

    def level_set(self, l, field, t: torch.Tensor):
        assert t.dtype == torch.float64 and t.is_cuda and t.is_contiguous() and tuple(t.shape) == self.level_shape(l)
        mg.mg_level_set(self.ctx, l, field, _ptr(t))

    def level_get(self, l, field) -> torch.Tensor:
        out = torch.empty(self.level_shape(l), dtype=torch.float64, device=self.device)
        mg.mg_level_get(self.ctx, l, field, _ptr(out))
        return out

    def timings(self):
        return mg.mg_get_timings(self.ctx, self.num_levels)

    def set_timing(self, on: bool):
        mg.mg_set_timing(self.ctx, on)

    def timing_records(self):
        """[(level, op, ms)] of every op timed since set_timing(True)."""
        return mg.mg_get_timing_records(self.ctx)

    def launches_per_vcycle(self) -> int:
        return mg.mg_vcycle_launches(self.ctx)

    def exchange_stats(self):
        return mg.mg_exchange_stats(self.ctx)

    def exchange_plan(self):
        """([exchanges per V-cycle per level], [bytes this rank sends per exchange per level])."""
        return mg.mg_exchange_plan(self.ctx, self.num_levels)

    def exchange_fused(self):
        """[exchanges per V-cycle per level fused into the pencil pass after them] (mg_exchange_fused)."""
        return mg.mg_exchange_fused(self.ctx, self.num_levels)

    def exchange_time(self, level, reps=20) -> float:
        """Device ms of one ghost exchange of x at `level` (collective over NCCL)."""
        return mg.mg_exchange_time(self.ctx, level, reps)


class LoopbackGroup:
    """world_size ranks of a proc_grid decomposition in one process on one GPU."""

    def __init__(self, n_local, proc_grid, num_levels=6, pre=12, post=12, bottom=100, ca_period=None, fusion=None,
                 ghost_mode=mg.MG_GHOST_AUTO, use_graph=True, bottom_mode=mg.MG_BOTTOM_AUTO, overlap=True, h0=0.0,
                 device=None, sweep_kernel=0, temporal_blocking=3, smoother=0, cheby_ratio=0, launch_pdl=0, bottom_solver=0,
                 bc=0, var_coef=0, brick_edge=0):
        self.device = torch.device("cuda", torch.cuda.current_device() if device is None else int(device))
        torch.cuda.set_device(self.device)
        self.n_local = tuple(int(v) for v in n_local)
        self.world_size = int(proc_grid[0] * proc_grid[1] * proc_grid[2])
        self.num_levels = int(num_levels)
        self.p = mg.params(self.n_local, proc_grid, num_levels, pre, post, bottom, ca_period, fusion, ghost_mode,
                           mg.MG_TRANSPORT_LOCAL, 1 if use_graph else 0, bottom_mode, 1 if overlap else 0, h0,
                           sweep_kernel, temporal_blocking, smoother, cheby_ratio, launch_pdl, bottom_solver, bc,
                           var_coef, brick_edge)
        per = (mg.mg_workspace_bytes(self.p, 0, self.world_size) + 255) & ~255
        self.ws = torch.empty(per * self.world_size + 256, dtype=torch.uint8, device=self.device)
        self.ws_ptr = (_ptr(self.ws) + 255) & ~255
        self.stream = torch.cuda.current_stream(self.device)
        self.g = mg.mg_group_setup(self.p, self.world_size, self.device.index, self.stream.cuda_stream, self.ws_ptr,
                                   per * self.world_size)

    @property
    def shape(self):
        return (self.n_local[2], self.n_local[1], self.n_local[0])

    def close(self):
        if getattr(self, "g", None):
            mg.mg_group_destroy(self.g)
            self.g = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_rhs(self, blocks):
        for r, b in enumerate(blocks):
            assert tuple(b.shape) == self.shape and b.is_cuda and b.dtype == torch.float64 and b.is_contiguous()
            mg.mg_group_set_rhs(self.g, r, _ptr(b))
        mg.mg_group_commit_rhs(self.g)

    def set_coefficients(self, blocks):
        for r, c in enumerate(blocks):
            assert tuple(c.shape) == self.shape and c.is_cuda and c.dtype == torch.float64 and c.is_contiguous()
            mg.mg_group_set_coefficients(self.g, r, _ptr(c))
        mg.mg_group_commit_coefficients(self.g)

    def set_solution(self, blocks=None):
        for r in range(self.world_size):
            if blocks is not None:
                b = blocks[r]
                assert tuple(b.shape) == self.shape and b.is_cuda and b.dtype == torch.float64 and b.is_contiguous()
            mg.mg_group_set_solution(self.g, r, None if blocks is None else _ptr(blocks[r]))

    def vcycle(self):
        mg.mg_group_vcycle(self.g)

    def residual_norm(self) -> float:
        return mg.mg_group_residual_norm(self.g)

    def get_solution(self, rank) -> torch.Tensor:
        out = torch.empty(self.shape, dtype=torch.float64, device=self.device)
        mg.mg_get_solution(mg.mg_group_ctx(self.g, rank), _ptr(out))
        return out

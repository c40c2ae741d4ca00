"""Thin ctypes binding of include/mg.h (argument marshalling only).

Every function here has the C name and forwards to libmg_b200.so; every step
of the V-cycle runs in the library's sm_100a kernels.  There is no CPU
fallback: if the library is missing or fails to load, ``lib()`` raises.
PyTorch is used only for device memory (the workspace and field tensors),
streams and (in the harness) process groups.
"""
from __future__ import annotations

import ctypes
import os

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(PKG, "libmg_b200.so")

MG_OK, MG_NOT_CONVERGED = 0, 1
MG_MAX_LEVELS = 16
MG_FUSION_AUTO, MG_FUSION_PAPER, MG_FUSION_SWEEP, MG_FUSION_FULL = 0, 1, 2, 3
MG_GHOST_AUTO, MG_GHOST_ALL = 0, 1
MG_TRANSPORT_AUTO, MG_TRANSPORT_NCCL, MG_TRANSPORT_LOCAL, MG_TRANSPORT_PEER = 0, 1, 2, 3
MG_PEER_BLOB_BYTES = 128
MG_BOTTOM_AUTO, MG_BOTTOM_SWEEPS, MG_BOTTOM_RESIDENT, MG_BOTTOM_CLUSTER, MG_BOTTOM_GRID = 0, 1, 2, 3, 4
MG_FIELD_X, MG_FIELD_B, MG_FIELD_R = 0, 1, 2
OP_NAMES = ["sweep", "applyOp", "smooth", "restriction", "interpolation", "initZero", "exchange", "bottom"]
MG_NUM_OPS = len(OP_NAMES)


class MGError(RuntimeError):
    def __init__(self, status: int, where: str, msg: str):
        super().__init__(f"{where} -> status {status}: {msg}")
        self.status = status


class mg_params(ctypes.Structure):
    _fields_ = [
        ("n_local", ctypes.c_int32 * 3),
        ("proc_grid", ctypes.c_int32 * 3),
        ("num_levels", ctypes.c_int32),
        ("pre_smooths", ctypes.c_int32),
        ("post_smooths", ctypes.c_int32),
        ("bottom_smooths", ctypes.c_int32),
        ("ca_period", ctypes.c_int32 * MG_MAX_LEVELS),
        ("fusion", ctypes.c_int32 * MG_MAX_LEVELS),
        ("ghost_mode", ctypes.c_int32),
        ("transport", ctypes.c_int32),
        ("use_graph", ctypes.c_int32),
        ("bottom_mode", ctypes.c_int32),
        ("overlap", ctypes.c_int32),
        ("sweep_kernel", ctypes.c_int32),
        ("temporal_blocking", ctypes.c_int32),
        ("smoother", ctypes.c_int32),
        ("cheby_ratio", ctypes.c_int32),
        ("launch_pdl", ctypes.c_int32),
        ("bottom_solver", ctypes.c_int32),
        ("bc", ctypes.c_int32),
        ("var_coef", ctypes.c_int32),
        ("brick_edge", ctypes.c_int32),
        ("h0", ctypes.c_double),
    ]


MG_BC_PERIODIC, MG_BC_DIRICHLET, MG_BC_NEUMANN = 0, 1, 2

_lib = None

_SIGS = {
    "mg_params_default": (None, [ctypes.POINTER(mg_params)]),
    "mg_workspace_bytes": (ctypes.c_int, [ctypes.POINTER(mg_params), ctypes.c_int32, ctypes.c_int32,
                                          ctypes.POINTER(ctypes.c_size_t)]),
    "mg_nccl_unique_id": (ctypes.c_int, [ctypes.c_char_p]),
    "mg_setup": (ctypes.c_int, [ctypes.POINTER(mg_params), ctypes.c_int32, ctypes.c_int32, ctypes.c_char_p,
                                ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t,
                                ctypes.POINTER(ctypes.c_void_p)]),
    "mg_set_rhs": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mg_set_rhs_host": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mg_set_solution": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mg_set_coefficients": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mg_get_solution": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mg_get_solution_host": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mg_vcycle": (ctypes.c_int, [ctypes.c_void_p]),
    "mg_residual_norm": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(ctypes.c_double)]),
    "mg_residual_norm_async": (ctypes.c_int, [ctypes.c_void_p]),
    "mg_get_timing_records": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(ctypes.c_int32),
                                             ctypes.POINTER(ctypes.c_double), ctypes.c_int32,
                                             ctypes.POINTER(ctypes.c_int32)]),
    "mg_residual_norm_wait": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(ctypes.c_double)]),
    "mg_solve": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_double, ctypes.c_int32, ctypes.POINTER(ctypes.c_int32),
                                ctypes.POINTER(ctypes.c_double)]),
    "mg_set_timing": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32]),
    "mg_get_timings": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(ctypes.c_double), ctypes.c_int32]),
    "mg_vcycle_launches": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(ctypes.c_int64)]),
    "mg_exchange_stats": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(ctypes.c_int64),
                                         ctypes.POINTER(ctypes.c_int64)]),
    "mg_peer_blob": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_char_p]),
    "mg_peer_connect": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_char_p]),
    "mg_layout_fused_pid": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.POINTER(ctypes.c_int64),
                                           ctypes.c_void_p]),
    "mg_exchange_fused": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.POINTER(ctypes.c_int64)]),
    "mg_exchange_plan": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.POINTER(ctypes.c_int64),
                                        ctypes.POINTER(ctypes.c_int64)]),
    "mg_exchange_time": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32,
                                        ctypes.POINTER(ctypes.c_double)]),
    "mg_destroy": (ctypes.c_int, [ctypes.c_void_p]),
    "mg_last_error": (ctypes.c_char_p, []),
    "mg_level_set": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p]),
    "mg_level_get": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p]),
    "mg_op_smooth": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32,
                                    ctypes.c_int32]),
    "mg_op_restrict": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32]),
    "mg_op_interp": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32]),
    "mg_op_bottom": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32]),
    "mg_sync": (ctypes.c_int, [ctypes.c_void_p]),
    "mg_group_setup": (ctypes.c_int, [ctypes.POINTER(mg_params), ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p,
                                      ctypes.c_void_p, ctypes.c_size_t, ctypes.POINTER(ctypes.c_void_p)]),
    "mg_group_ctx": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.POINTER(ctypes.c_void_p)]),
    "mg_group_vcycle": (ctypes.c_int, [ctypes.c_void_p]),
    "mg_group_residual_norm": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(ctypes.c_double)]),
    "mg_group_set_rhs": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p]),
    "mg_group_commit_rhs": (ctypes.c_int, [ctypes.c_void_p]),
    "mg_group_set_coefficients": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p]),
    "mg_group_commit_coefficients": (ctypes.c_int, [ctypes.c_void_p]),
    "mg_group_set_solution": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p]),
    "mg_group_destroy": (ctypes.c_int, [ctypes.c_void_p]),
    "mg_layout_create": (ctypes.c_int, [ctypes.POINTER(mg_params), ctypes.c_int32, ctypes.c_int32,
                                        ctypes.POINTER(ctypes.c_void_p)]),
    "mg_layout_level_info": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.POINTER(ctypes.c_int64)]),
    "mg_layout_adjacency": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p]),
    "mg_layout_coords": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p]),
    "mg_layout_parent": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p]),
    "mg_layout_plan": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p]),
    "mg_layout_mirror": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p]),
    "mg_layout_pass_plan": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p,
                                           ctypes.c_void_p, ctypes.c_void_p]),
    "mg_layout_repl": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                      ctypes.c_void_p]),
    "mg_layout_vcycle_launches": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.POINTER(ctypes.c_int64)]),
    "mg_layout_exchange_plan": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.POINTER(ctypes.c_int64),
                                               ctypes.POINTER(ctypes.c_int64)]),
    "mg_layout_destroy": (ctypes.c_int, [ctypes.c_void_p]),
}


def lib():
    """Load libmg_b200.so (raises if it is missing: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built: run __graft_entry__.build() (no CPU fallback exists)")
        # torch first, so the NCCL torch bundles is the libnccl.so.2 in the process
        try:
            import torch  # noqa: F401
        except Exception:
            pass
        L = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in _SIGS.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def header_symbols():
    return list(_SIGS)


def check(status: int, where: str) -> int:
    if status < 0:
        raise MGError(status, where, lib().mg_last_error().decode())
    return status


def params(n_local, proc_grid=(1, 1, 1), num_levels=6, pre=12, post=12, bottom=100, ca_period=None, fusion=None,
           ghost_mode=MG_GHOST_AUTO, transport=MG_TRANSPORT_AUTO, use_graph=1, bottom_mode=MG_BOTTOM_AUTO,
           overlap=1, h0=0.0, sweep_kernel=0, temporal_blocking=3, smoother=0, cheby_ratio=0, launch_pdl=0, bottom_solver=0,
           bc=0, var_coef=0, brick_edge=0) -> mg_params:
    p = mg_params()
    lib().mg_params_default(ctypes.byref(p))
    p.n_local[:] = [int(v) for v in n_local]
    p.proc_grid[:] = [int(v) for v in proc_grid]
    p.num_levels = int(num_levels)
    p.pre_smooths, p.post_smooths, p.bottom_smooths = int(pre), int(post), int(bottom)
    for l in range(MG_MAX_LEVELS):
        p.ca_period[l] = 0 if ca_period is None else int(ca_period[l] if isinstance(ca_period, (list, tuple))
                                                          else ca_period)
        p.fusion[l] = 0 if fusion is None else int(fusion[l] if isinstance(fusion, (list, tuple)) else fusion)
    p.ghost_mode, p.transport, p.use_graph = int(ghost_mode), int(transport), int(use_graph)
    p.bottom_mode, p.overlap, p.h0 = int(bottom_mode), int(overlap), float(h0)
    p.sweep_kernel = int(sweep_kernel)
    p.temporal_blocking = int(temporal_blocking)
    p.smoother, p.cheby_ratio = int(smoother), int(cheby_ratio)
    p.launch_pdl = int(launch_pdl)
    p.bottom_solver = int(bottom_solver)
    p.bc, p.var_coef = int(bc), int(var_coef)
    p.brick_edge = int(brick_edge)
    return p


# ----------------------------------------------------------------- C names
def mg_workspace_bytes(p: mg_params, rank: int = 0, world_size: int = 1) -> int:
    out = ctypes.c_size_t()
    check(lib().mg_workspace_bytes(ctypes.byref(p), rank, world_size, ctypes.byref(out)), "mg_workspace_bytes")
    return out.value


def mg_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    check(lib().mg_nccl_unique_id(buf), "mg_nccl_unique_id")
    return buf.raw


def mg_setup(p, rank, world_size, nccl_id, device, stream, workspace_ptr, ws_bytes):
    ctx = ctypes.c_void_p()
    check(lib().mg_setup(ctypes.byref(p), rank, world_size, nccl_id, device, stream, workspace_ptr, ws_bytes,
                         ctypes.byref(ctx)), "mg_setup")
    return ctx


def mg_set_rhs(ctx, b_ptr):
    return check(lib().mg_set_rhs(ctx, b_ptr), "mg_set_rhs")


def mg_set_rhs_host(ctx, b_host_ptr):
    return check(lib().mg_set_rhs_host(ctx, b_host_ptr), "mg_set_rhs_host")


def mg_set_coefficients(ctx, c_ptr):
    return check(lib().mg_set_coefficients(ctx, c_ptr), "mg_set_coefficients")


def mg_set_solution(ctx, x_ptr):
    return check(lib().mg_set_solution(ctx, x_ptr), "mg_set_solution")


def mg_get_solution(ctx, x_ptr):
    return check(lib().mg_get_solution(ctx, x_ptr), "mg_get_solution")


def mg_get_solution_host(ctx, x_host_ptr):
    return check(lib().mg_get_solution_host(ctx, x_host_ptr), "mg_get_solution_host")


def mg_vcycle(ctx):
    return check(lib().mg_vcycle(ctx), "mg_vcycle")


def mg_residual_norm(ctx) -> float:
    out = ctypes.c_double()
    check(lib().mg_residual_norm(ctx, ctypes.byref(out)), "mg_residual_norm")
    return out.value


def mg_residual_norm_async(ctx) -> None:
    check(lib().mg_residual_norm_async(ctx), "mg_residual_norm_async")


def mg_residual_norm_wait(ctx) -> float:
    out = ctypes.c_double()
    check(lib().mg_residual_norm_wait(ctx, ctypes.byref(out)), "mg_residual_norm_wait")
    return out.value


def mg_solve(ctx, tol=1e-10, max_cycles=20):
    cyc, fin = ctypes.c_int32(), ctypes.c_double()
    st = check(lib().mg_solve(ctx, tol, max_cycles, ctypes.byref(cyc), ctypes.byref(fin)), "mg_solve")
    return st, cyc.value, fin.value


def mg_set_timing(ctx, enabled: bool):
    return check(lib().mg_set_timing(ctx, 1 if enabled else 0), "mg_set_timing")


def mg_get_timings(ctx, num_levels: int):
    n = num_levels * MG_NUM_OPS
    buf = (ctypes.c_double * n)()
    check(lib().mg_get_timings(ctx, buf, n), "mg_get_timings")
    return [[buf[l * MG_NUM_OPS + o] for o in range(MG_NUM_OPS)] for l in range(num_levels)]


def mg_get_timing_records(ctx):
    """[(level, op, ms)] of every timed op since mg_set_timing (issue order)."""
    n = ctypes.c_int32()
    check(lib().mg_get_timing_records(ctx, None, None, 0, ctypes.byref(n)), "mg_get_timing_records")
    cap = n.value
    slots = (ctypes.c_int32 * max(cap, 1))()
    ms = (ctypes.c_double * max(cap, 1))()
    check(lib().mg_get_timing_records(ctx, slots, ms, cap, ctypes.byref(n)), "mg_get_timing_records")
    return [(slots[i] // MG_NUM_OPS, slots[i] % MG_NUM_OPS, ms[i]) for i in range(min(cap, n.value))]


def mg_vcycle_launches(ctx) -> int:
    out = ctypes.c_int64()
    check(lib().mg_vcycle_launches(ctx, ctypes.byref(out)), "mg_vcycle_launches")
    return out.value


def mg_exchange_stats(ctx):
    b, m = ctypes.c_int64(), ctypes.c_int64()
    check(lib().mg_exchange_stats(ctx, ctypes.byref(b), ctypes.byref(m)), "mg_exchange_stats")
    return b.value, m.value


def mg_peer_blob(ctx) -> bytes:
    buf = ctypes.create_string_buffer(MG_PEER_BLOB_BYTES)
    check(lib().mg_peer_blob(ctx, buf), "mg_peer_blob")
    return buf.raw


def mg_peer_connect(ctx, blobs: bytes):
    return check(lib().mg_peer_connect(ctx, blobs), "mg_peer_connect")


def mg_exchange_plan(ctx, num_levels):
    ex = (ctypes.c_int64 * num_levels)()
    by = (ctypes.c_int64 * num_levels)()
    check(lib().mg_exchange_plan(ctx, num_levels, ex, by), "mg_exchange_plan")
    return list(ex), list(by)


def mg_exchange_fused(ctx, num_levels):
    fu = (ctypes.c_int64 * num_levels)()
    check(lib().mg_exchange_fused(ctx, num_levels, fu), "mg_exchange_fused")
    return list(fu)


def mg_exchange_time(ctx, level, reps=20):
    ms = ctypes.c_double()
    check(lib().mg_exchange_time(ctx, level, reps, ctypes.byref(ms)), "mg_exchange_time")
    return ms.value


def mg_destroy(ctx):
    return check(lib().mg_destroy(ctx), "mg_destroy")


def mg_level_set(ctx, level, field, ptr):
    return check(lib().mg_level_set(ctx, level, field, ptr), "mg_level_set")


def mg_level_get(ctx, level, field, ptr):
    return check(lib().mg_level_get(ctx, level, field, ptr), "mg_level_get")


def mg_op_smooth(ctx, level, n, write_r, fusion=MG_FUSION_SWEEP):
    return check(lib().mg_op_smooth(ctx, level, n, 1 if write_r else 0, fusion), "mg_op_smooth")


def mg_op_restrict(ctx, level):
    return check(lib().mg_op_restrict(ctx, level), "mg_op_restrict")


def mg_op_interp(ctx, level):
    return check(lib().mg_op_interp(ctx, level), "mg_op_interp")


def mg_op_bottom(ctx, level, n):
    return check(lib().mg_op_bottom(ctx, level, n), "mg_op_bottom")


def mg_sync(ctx):
    return check(lib().mg_sync(ctx), "mg_sync")


def mg_group_setup(p, world_size, device, stream, workspace_ptr, ws_bytes):
    g = ctypes.c_void_p()
    check(lib().mg_group_setup(ctypes.byref(p), world_size, device, stream, workspace_ptr, ws_bytes,
                               ctypes.byref(g)), "mg_group_setup")
    return g


def mg_group_ctx(g, rank):
    c = ctypes.c_void_p()
    check(lib().mg_group_ctx(g, rank, ctypes.byref(c)), "mg_group_ctx")
    return c


def mg_group_vcycle(g):
    return check(lib().mg_group_vcycle(g), "mg_group_vcycle")


def mg_group_residual_norm(g) -> float:
    out = ctypes.c_double()
    check(lib().mg_group_residual_norm(g, ctypes.byref(out)), "mg_group_residual_norm")
    return out.value


def mg_group_set_rhs(g, rank, ptr):
    return check(lib().mg_group_set_rhs(g, rank, ptr), "mg_group_set_rhs")


def mg_group_commit_rhs(g):
    return check(lib().mg_group_commit_rhs(g), "mg_group_commit_rhs")


def mg_group_set_coefficients(g, rank, ptr):
    return check(lib().mg_group_set_coefficients(g, rank, ptr), "mg_group_set_coefficients")


def mg_group_commit_coefficients(g):
    return check(lib().mg_group_commit_coefficients(g), "mg_group_commit_coefficients")


def mg_group_set_solution(g, rank, ptr):
    return check(lib().mg_group_set_solution(g, rank, ptr), "mg_group_set_solution")


def mg_group_destroy(g):
    return check(lib().mg_group_destroy(g), "mg_group_destroy")


# ------------------------------------------------------- layout (host only)
class Layout:
    """Host-side brick layout tables of one rank (no GPU needed)."""

    def __init__(self, p: mg_params, rank: int = 0, world_size: int = 1):
        import numpy as np

        self._np = np
        self.p = p
        self.h = ctypes.c_void_p()
        check(lib().mg_layout_create(ctypes.byref(p), rank, world_size, ctypes.byref(self.h)), "mg_layout_create")

    def __del__(self):
        if getattr(self, "h", None):
            lib().mg_layout_destroy(self.h)
            self.h = None

    def info(self, level):
        buf = (ctypes.c_int64 * 16)()
        check(lib().mg_layout_level_info(self.h, level, buf), "mg_layout_level_info")
        v = list(buf)
        return {"n": v[0:3], "nb": v[3:6], "ghost": v[6:9], "owned": v[9], "interior": v[10], "nghost": v[11],
                "alloc": v[12], "send_runs": v[13], "recv_runs": v[14], "zero_brick": v[15]}

    def repl(self):
        """Replicated bottom maps: None, or (gb_src, gb_mine, gb_adj) (see mg_layout_repl)."""
        np = self._np
        info = (ctypes.c_int64 * 2)()
        check(lib().mg_layout_repl(self.h, info, None, None, None), "mg_layout_repl")
        if info[0] == 0:
            return None
        src = np.zeros(info[0], dtype=np.int32)
        mine = np.zeros(info[1], dtype=np.int32)
        adj = np.zeros((info[0], 8), dtype=np.int32)
        check(lib().mg_layout_repl(self.h, info, src.ctypes.data, mine.ctypes.data, adj.ctypes.data), "mg_layout_repl")
        return src, mine, adj

    def mirror(self, level):
        """[n][3] (ghost brick, source brick, reflected-axes mask) of a non-periodic bc (reading A22)."""
        np = self._np
        n = ctypes.c_int64()
        check(lib().mg_layout_mirror(self.h, level, ctypes.byref(n), None), "mg_layout_mirror")
        a = np.zeros((n.value, 3), dtype=np.int32)
        if n.value:
            check(lib().mg_layout_mirror(self.h, level, ctypes.byref(n), a.ctypes.data), "mg_layout_mirror")
        return a

    def adjacency(self, level):
        inf = self.info(level)
        a = self._np.zeros((inf["owned"] + inf["nghost"], 8), dtype=self._np.int32)
        check(lib().mg_layout_adjacency(self.h, level, a.ctypes.data), "mg_layout_adjacency")
        return a

    def coords(self, level):
        inf = self.info(level)
        a = self._np.zeros((inf["owned"] + inf["nghost"], 3), dtype=self._np.int32)
        check(lib().mg_layout_coords(self.h, level, a.ctypes.data), "mg_layout_coords")
        return a

    def parent(self, level):
        inf = self.info(level)
        a = self._np.zeros(inf["owned"] + inf["nghost"], dtype=self._np.int32)
        check(lib().mg_layout_parent(self.h, level, a.ctypes.data), "mg_layout_parent")
        return a

    def fused_pid(self, level):
        """The fused exchange's source table of a level (mg_layout_fused_pid): int32 [chunks][16], or None."""
        n = ctypes.c_int64()
        check(lib().mg_layout_fused_pid(self.h, level, ctypes.byref(n), None), "mg_layout_fused_pid")
        if n.value == 0:
            return None
        a = self._np.zeros(n.value, dtype=self._np.int32)
        check(lib().mg_layout_fused_pid(self.h, level, ctypes.byref(n), a.ctypes.data), "mg_layout_fused_pid")
        return a.reshape(-1, 16)

    def pass_plans(self, level):
        """Two-sweep pass plans of a level: [(kind, b0, b1, meta int32 array, ctas int32 [n][2], part)]."""
        np = self._np
        out = []
        for idx in range(64):
            info = (ctypes.c_int64 * 6)()
            if lib().mg_layout_pass_plan(self.h, level, idx, info, None, None) != 0:
                break
            meta = np.zeros(max(info[3], 1), dtype=np.int32)
            ctas = np.zeros(max(info[4], 2), dtype=np.int32)
            check(lib().mg_layout_pass_plan(self.h, level, idx, info, meta.ctypes.data, ctas.ctypes.data),
                  "mg_layout_pass_plan")
            out.append((info[0], info[1], info[2], meta[:info[3]], ctas[:info[4]].reshape(-1, 2), info[5]))
        return out

    def exchange_plan(self):
        """(exchanges per level, bytes per x-exchange per level) of a fresh context's first V-cycle."""
        n = self.p.num_levels
        ex, by = (ctypes.c_int64 * n)(), (ctypes.c_int64 * n)()
        check(lib().mg_layout_exchange_plan(self.h, n, ex, by), "mg_layout_exchange_plan")
        return list(ex), list(by)

    def vcycle_launches(self, local_exchange=True) -> int:
        """Own kernel launches of one V-cycle (mg_layout_vcycle_launches)."""
        out = ctypes.c_int64()
        check(lib().mg_layout_vcycle_launches(self.h, 1 if local_exchange else 0, ctypes.byref(out)),
              "mg_layout_vcycle_launches")
        return out.value

    def plan(self, level, which):
        inf = self.info(level)
        n = inf["recv_runs"] if which else inf["send_runs"]
        a = self._np.zeros((n, 6), dtype=self._np.int64)
        if n:
            check(lib().mg_layout_plan(self.h, level, which, a.ctypes.data), "mg_layout_plan")
        return a

#!/usr/bin/env python
"""bench.py -- V-cycle DOF/s and finest-level smoother HBM GB/s on B200.

Workload (BASELINE.json configs[3] at N GPUs, configs[2]'s size at N=1):
512^3 FP64 Poisson per GPU, 8^3 bricks, L = 6 levels (512 -> 16), 12 pre /
12 post smooths, 100 bottom sweeps, weak scaling with a 3D
decomposition (1x1x1, 2x1x1, 2x2x1, 2x2x2).  b = sin(2 pi x) sin(2 pi y)
sin(2 pi z), x0 = 0.  One "step" = one V-cycle (Alg 2).

Usage:  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
        torchrun --nproc-per-node N bench.py --gpus N ...   (one rank per GPU, NCCL)
Prints ONE JSON line on rank 0 (contract in DESIGN.md "Measurement").
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "V-cycle DOF/s and finest-level smoother HBM GB/s (fraction of 8 TB/s) at 1/2/4/8 B200"
PROC_GRIDS = {1: (1, 1, 1), 2: (2, 1, 1), 4: (2, 2, 1), 8: (2, 2, 2)}
# algorithmic bytes per fine point (Table IV)
B_SWEEP = 24.0          # fused sweep: read x, b; write x'
B_SWEEP_R = 32.0        # + write r
B_COARSE_PER_FINE = 1.0  # fused restriction output / interpolation input (8 B per coarse point)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--n", "--size", dest="n", type=int, default=512,
                    help="cells per GPU per axis (--size under torchrun: '--n' is ambiguous to its parser)")
    ap.add_argument("--levels", type=int, default=6)
    ap.add_argument("--pre", type=int, default=12)
    ap.add_argument("--post", type=int, default=12)
    ap.add_argument("--bottom", type=int, default=100)
    ap.add_argument("--ca-period", type=int, default=0)
    ap.add_argument("--fusion", type=int, default=0)
    ap.add_argument("--ghost-all", action="store_true", help="self-exchange ghost shell on every axis")
    ap.add_argument("--transport", choices=["auto", "peer", "nccl", "local"], default="auto",
                    help="ghost exchange transport (auto: peer memory (CUDA IPC + device flags) between processes, "
                         "device copies for a one-rank self-exchange; peer / nccl: that transport even to itself)")
    ap.add_argument("--no-graph", action="store_true")
    ap.add_argument("--no-overlap", action="store_true")
    ap.add_argument("--tb", type=int, default=3,
                    help="temporal blocking (two sweeps per HBM pass): 3 = 2x2-brick pencils, two-warp CTAs (sweep2p.cu, "
                         "default), 1 = one-brick CTA streams (sweep2.cu), 0 = off")
    ap.add_argument("--smoother", type=int, default=0,
                    help="0 damped Jacobi (the paper), 1 Chebyshev, 2 red-black Gauss-Seidel (N4 variants)")
    ap.add_argument("--cheby-ratio", type=int, default=0, help="Chebyshev smoothing interval [mu_max/ratio, mu_max]")
    ap.add_argument("--no-pdl", action="store_true", help="launch kernels without programmatic dependent launch")
    ap.add_argument("--bottom-solver", type=int, default=0, help="0 Jacobi smooths (the paper), 1 CG (variant)")
    ap.add_argument("--bottom-mode", type=int, default=0,
                    help="0 auto, 1 per-sweep launches, 2 resident bottom, 3 cluster coarse solve, 4 grid coarse solve")
    ap.add_argument("--bc", type=int, default=0, help="variant (reading A22): 0 periodic (the paper), 1 Dirichlet, 2 Neumann")
    ap.add_argument("--var-coef", action="store_true", help="variant (reading A23): div(c grad x), smooth c")
    ap.add_argument("--brick-edge", type=int, default=0, help="variant: 4 = 4^3 bricks (P:L154 Sunspot)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--ref-n", type=int, default=0, help="reference arm: grid side of the bounded sample")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--quiet", action="store_true")
    return ap.parse_args()


def host_cores():
    """Cores this process may run on (the oracle's OpenMP threads for the CPU legs)."""
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def workload_name(a, pg):
    e = a.brick_edge or 8
    var = "".join([{0: "", 1: ", Dirichlet", 2: ", Neumann"}[a.bc], ", variable coefficients" if a.var_coef else ""])
    return (f"{a.n}^3 FP64 Poisson per GPU, {e}^3 bricks, L={a.levels} ({a.n}->{a.n >> (a.levels - 1)}), "
            f"{a.pre}/{a.post}/{a.bottom} smooths, 3D decomposition {pg[0]}x{pg[1]}x{pg[2]}{var}")


# ------------------------------------------------------------------ clocks
class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.proc = None
        self.path = None

    def start(self):
        try:
            fd, self.path = tempfile.mkstemp(suffix=".csv")
            os.close(fd)
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if not self.proc:
            return None
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        rows = []
        for line in open(self.path):
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                rows.append((float(parts[1]), float(parts[2]), float(parts[3]), parts[5:9]))
            except ValueError:
                continue
        os.unlink(self.path)
        if not rows:
            return None
        load = [r for r in rows if r[2] > 200.0] or rows
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in load for i, v in enumerate(r[3]) if v.lower() == "active"})
        return {"sm_mhz": statistics.median(r[0] for r in load), "sm_max_mhz": max(r[1] for r in rows),
                "reasons": reasons, "samples": len(rows), "samples_under_load": len(load),
                "power_w_max": max(r[2] for r in rows)}


def measured_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        d = json.load(open(path))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, STREAM-style copy)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def ncu_traffic(n, kernel):
    """Per-launch DRAM bytes of the level-0 pass kernel from the committed ncu --set full summary
    (None unless that summary is of the same kernel at the same size)."""
    path = os.path.join(ROOT, "profiles", "ncu_sweep_summary.json")
    if not os.path.exists(path):
        return None
    try:
        d = json.load(open(path))
        if int(d.get("n", -1)) == n and d.get("kernel", "").split("<")[0].split()[-1] == kernel:
            return float(d["dram_bytes_per_launch"])
    except Exception:
        pass
    return None


# ------------------------------------------------------------------ oracle timing
def oracle_dofs(n, levels, pre, post, bottom, seconds, min_cycles=1, max_cycles=1000, threads=None):
    """Time the CPU oracle (as it stands) running V-cycles on an n^3 grid."""
    import mg_inputs
    import oracle

    oracle.build()
    # the host's cores by default (torchrun sets OMP_NUM_THREADS=1 per process)
    oracle.set_threads(threads or host_cores())
    b = mg_inputs.sin_rhs((n, n, n))
    m = oracle.OracleMG((n, n, n), levels, pre, post, bottom)
    m.set_b(b)
    m.set_x(None)
    t0 = time.perf_counter()
    c = 0
    while c < min_cycles or (time.perf_counter() - t0 < seconds and c < max_cycles):
        m.vcycle()
        c += 1
    dt = time.perf_counter() - t0
    m.close()
    return n**3 * c / dt, c, dt, oracle.get_threads()


def cpu_baseline(a):
    # estimate with one 256^3 cycle, use the real workload size when it fits the budget
    small = min(a.n, 256)
    lv_small = max(1, min(a.levels, (small // 8).bit_length()))
    v, c, dt, cores = oracle_dofs(small, lv_small, a.pre, a.post, a.bottom, 0.0)
    est_full = dt * (a.n / small) ** 3
    if a.n != small and est_full <= a.cpu_seconds:
        v, c, dt, cores = oracle_dofs(a.n, a.levels, a.pre, a.post, a.bottom, a.cpu_seconds)
        sample = f"{c} oracle V-cycle(s) of the {a.n}^3 workload itself (L={a.levels}), {dt:.1f} s"
    else:
        lv = lv_small
        v, c2, dt2, cores = oracle_dofs(small, lv, a.pre, a.post, a.bottom, a.cpu_seconds)
        sample = (f"{c2} oracle V-cycle(s) on a {small}^3 grid (L={lv}, same sweeps), {dt2:.1f} s; "
                  f"DOF/s of that sample")
    # the same oracle on one core (both core counts), on a 256^3 sample (one cycle
    # of the 512^3 workload would take ~30 s on one core)
    v1, c1, dt1, _ = oracle_dofs(small, lv_small, a.pre, a.post, a.bottom, 0.0, threads=1)
    single = {"value": v1, "unit": "DOF/s", "cores": 1,
              "sample": f"{c1} oracle V-cycle(s) on a {small}^3 grid (L={lv_small}) on one thread, {dt1:.1f} s"}
    return {"value": v, "unit": "DOF/s", "cores": cores, "kind": "oracle", "sample": sample, "single_thread": single}


def run_reference(a, rank, world):
    """--impl reference: the CPU oracle as it stands on the host cores (rank 0 only)."""
    if rank != 0:
        return
    import oracle

    oracle.build()
    oracle.set_threads(host_cores())
    import mg_inputs

    def setup(n, lv):
        m = oracle.OracleMG((n, n, n), lv, a.pre, a.post, a.bottom)
        m.set_b(mg_inputs.sin_rhs((n, n, n)))
        m.set_x(None)
        return m

    # the workload itself (512^3 per rank, L = 6: about 2 s per oracle cycle on 16 cores); a 256^3
    # sample only if the first (warm-up) cycle says the run would not end within ~5 minutes
    n = a.ref_n or a.n
    lv = a.levels if n == a.n else max(1, min(a.levels, (n // 8).bit_length()))
    m = setup(n, lv)
    t0 = time.perf_counter()
    m.vcycle()
    t1 = time.perf_counter() - t0
    if not a.ref_n and t1 * (a.steps + a.warmup) > 300.0 and n > 256:
        m.close()
        n = 256
        lv = max(1, min(a.levels, (n // 8).bit_length()))
        m = setup(n, lv)
        m.vcycle()
    for _ in range(a.warmup - 1):
        m.vcycle()
    t0 = time.perf_counter()
    for _ in range(a.steps):
        m.vcycle()
    dt = time.perf_counter() - t0
    value = n**3 * a.steps / dt
    pg = PROC_GRIDS.get(a.gpus, (1, 1, 1))
    sample = (f"each step = one oracle V-cycle of the {n}^3 workload (L={lv}, {a.pre}/{a.post}/{a.bottom})"
              if n == a.n and lv == a.levels else
              f"each step = one oracle V-cycle on a {n}^3 grid (L={lv}, {a.pre}/{a.post}/{a.bottom}), bounded sample")
    line = {"metric": METRIC, "value": value, "unit": "DOF/s", "n_gpus": a.gpus, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": dt / a.steps * 1e3, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
            "config": {"workload": workload_name(a, pg) if n == a.n else
                       f"{n}^3 sample of: " + workload_name(a, pg), "sample_grid": n, "levels": lv},
            "cpu_baseline": {"value": value, "unit": "DOF/s", "cores": oracle.get_threads(), "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": value, "unit": "DOF/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ exchanges
NVLINK_GBS = 900.0  # NVLink 5: 900 GB/s per direction per GPU (B200_PROFILING.md)


def exchange_block(m, a, world, max_over_ranks, tm, ninst):
    from paper_conf_sc_antepara0jh24_b200 import mg

    """Per level: ghost exchanges per V-cycle, bytes per exchange, device time of one exchange (the
    V-cycle's own transport, back to back, max over ranks), achieved GB/s and its fraction of the
    NVLink per-direction bandwidth (between processes) -- plus the latency / bandwidth fit
    t = alpha + bytes / beta over the levels (P:L216-236, N3) and the Table-II-style share of the
    exchanges in the level time (P:L198-206)."""
    counts, nbytes = m.exchange_plan()
    fused = m.exchange_fused()  # of which: fused into the pencil pass after them (no exchange kernel)
    if not any(nbytes):
        return {"levels": [], "note": "no ghost shell (one rank, periodic wrap): no exchanges"}
    transport = {mg.MG_TRANSPORT_NCCL: "nccl", mg.MG_TRANSPORT_PEER: "peer memory (CUDA IPC, device flags)"}.get(
        m.transport, "peer memory (CUDA IPC, device flags)" if world > 1 else "local device copies")
    out = []
    for l, (c, b) in enumerate(zip(counts, nbytes)):
        if b <= 0:
            continue
        t = max_over_ranks(m.exchange_time(l, 20))
        gbs = b / (t / 1e3) / 1e9 if t > 0 else None
        lvl_ms = sum(tm[l]) / ninst if l < len(tm) else None
        out.append({"level": l, "exchanges_per_cycle": c, "fused_into_pencil_pass": fused[l],
                    "bytes_per_exchange": b, "ms_per_exchange": t,
                    "gbs": gbs, "frac_of_nvlink_900": (gbs / NVLINK_GBS) if (gbs and world > 1) else None,
                    "ms_per_cycle_if_serial": (c - fused[l]) * t,
                    "share_of_level_time": ((c - fused[l]) * t / lvl_ms) if lvl_ms else None})
    fit = None
    pts = [(d["bytes_per_exchange"], d["ms_per_exchange"]) for d in out if d["ms_per_exchange"] > 0]
    if len(pts) >= 2:
        import numpy as np

        X = np.array([[1.0, p[0]] for p in pts])
        y = np.array([p[1] for p in pts])
        (alpha, inv_beta), *_ = np.linalg.lstsq(X, y, rcond=None)
        fit = {"alpha_us": alpha * 1e3, "beta_gbs": (1.0 / inv_beta / 1e6) if inv_beta > 0 else None,
               "points": len(pts)}
    return {"transport": transport, "levels": out, "fit": fit,
            "link": "NVLink 5, 900 GB/s per direction" if world > 1 else "self-exchange on one GPU (no link)"}


# ------------------------------------------------------------------ GPU arm
def main():
    a = parse()
    rank, world, local = dist_env()
    if a.impl == "reference":
        run_reference(a, rank, world)
        return
    import numpy as np
    import torch
    import torch.distributed as dist

    import mg_inputs
    from paper_conf_sc_antepara0jh24_b200 import mg
    from paper_conf_sc_antepara0jh24_b200.solver import Multigrid

    if world != a.gpus:
        a.gpus = world if world > 1 else a.gpus
    # MG_BENCH_SHARED_GPU=1 (rehearsal of the multi-rank path on a one-GPU box, not a measurement):
    # ranks share the visible GPUs round-robin, torch.distributed runs on gloo (the library exchanges
    # ghosts over peer memory, which CUDA IPC allows between processes on one device)
    shared = os.environ.get("MG_BENCH_SHARED_GPU") == "1"
    if shared:
        local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    pg = PROC_GRIDS[world]
    n = a.n
    m = Multigrid((n, n, n), pg, a.levels, a.pre, a.post, a.bottom, ca_period=a.ca_period, fusion=a.fusion,
                  ghost_mode=1 if a.ghost_all else 0, use_graph=not a.no_graph, overlap=not a.no_overlap,
                  rank=rank, world_size=world, device=local, temporal_blocking=a.tb, smoother=a.smoother,
                  cheby_ratio=a.cheby_ratio, launch_pdl=2 if a.no_pdl else 0,
                  bottom_mode=a.bottom_mode, bottom_solver=a.bottom_solver, bc=a.bc,
                  var_coef=1 if a.var_coef else 0, brick_edge=a.brick_edge,
                  transport={"auto": mg.MG_TRANSPORT_AUTO, "nccl": mg.MG_TRANSPORT_NCCL,
                             "local": mg.MG_TRANSPORT_LOCAL, "peer": mg.MG_TRANSPORT_PEER}[a.transport])
    gshape = (n * pg[2], n * pg[1], n * pg[0])
    if a.bc == 1:  # the lowest Dirichlet mode (the sin b of P:L148 is not zero on the faces)
        b_host = torch.from_numpy(mg_inputs.local_block(mg_inputs.dirichlet_sin_rhs(gshape), rank, pg)).pin_memory()
    else:
        b_host = torch.from_numpy(mg_inputs.local_sin_rhs(gshape, rank, pg)).pin_memory()
    if a.var_coef:
        m.set_coefficients(torch.from_numpy(mg_inputs.local_block(mg_inputs.smooth_coef(gshape), rank, pg)).to(dev))
    b_dev = b_host.to(dev)
    m.set_rhs(b_dev)
    m.set_solution(None)
    s = m.stream

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(v):
        if world > 1:
            t = torch.tensor([v], dtype=torch.float64, device="cpu" if shared else dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            return float(t.item())
        return v

    # ---- warm-up (also captures the CUDA graph)
    for _ in range(a.warmup):
        m.vcycle()
    barrier()
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    # ---- timed region: K V-cycles, device-timed with events on the library's stream
    barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(a.steps):
        m.vcycle()
    e1.record(s)
    barrier()
    t_ms = max_over_ranks(e0.elapsed_time(e1))
    clk = clocks.stop()
    dofs = world * n**3 * a.steps / (t_ms / 1e3)
    norm = m.residual_norm()

    # ---- instrumented pass: per (level, op) device times with CUDA events (no graph)
    m.set_timing(True)
    ninst = max(1, min(a.steps, 5))
    for _ in range(ninst):
        m.vcycle()
    torch.cuda.synchronize()
    tm = m.timings()
    recs = m.timing_records()  # (mg_set_timing clears them)
    m.set_timing(False)
    nsweep0 = a.pre + a.post
    # every level-0 pass of the instrumented cycles, from the per-op records (two-sweep passes and any
    # single sweeps alike; the interpolation is its own op where the pencil passes run)
    passes0 = [ms for (lv, op, ms) in recs if lv == 0 and op == mg.OP_NAMES.index("sweep")]
    sweep0_ms = sum(passes0) / ninst
    npass0 = round(len(passes0) / ninst)
    launch_ms = sweep0_ms / npass0
    interp_fused = tm[0][mg.OP_NAMES.index("interpolation")] == 0
    # algorithmic bytes of the level-0 passes of one V-cycle (24 B/pt each: read x, b; write x'),
    # + 1 B/pt for the fused restriction output (and the fused interpolation input, if fused)
    fusion0 = a.fusion or mg.MG_FUSION_FULL
    pts = n**3
    bytes0 = pts * (B_SWEEP * npass0 + (2 if interp_fused else 1) * B_COARSE_PER_FINE)
    if fusion0 != mg.MG_FUSION_FULL:
        bytes0 = pts * (B_SWEEP * (npass0 - 1) + B_SWEEP_R)
    achieved = bytes0 / (sweep0_ms / 1e3) / 1e9
    # the same level-0 work expressed as one-sweep-per-pass traffic (what the sweeps would move unblocked)
    sweep_equiv = pts * (B_SWEEP * nsweep0 + 2 * B_COARSE_PER_FINE) / (sweep0_ms / 1e3) / 1e9
    peak, peak_src = measured_peaks()
    pass_kernel = {0: "sweep_col_kernel", 1: "sweep2_kernel"}.get(
        a.tb, "sweep2p_kernel")
    traffic = ncu_traffic(n, pass_kernel)
    levels = []
    total_inst = sum(sum(r) for r in tm) / ninst
    for l, row in enumerate(tm):
        nl = n >> l
        d = {"level": l, "n": nl, "ms": {k: round(v / ninst, 4) for k, v in zip(mg.OP_NAMES, row) if v > 0}}
        if row[0] > 0 and l < a.levels - 1:
            lb = nl**3 * (B_SWEEP * (a.pre + a.post) + (2 if fusion0 == mg.MG_FUSION_FULL else 8) * B_COARSE_PER_FINE)
            d["sweep_equivalent_gbs"] = round(lb / (row[0] / ninst / 1e3) / 1e9, 1)  # 24 B/pt per sweep
        levels.append(d)

    # ---- e2e: public API with host buffers (H2D of b, V-cycle, D2H of the norm) per step
    e2e = None
    if not a.no_e2e:
        ke = max(3, a.steps)  # the same K steps as the device-timed loop (the pipeline's last V-cycle is its tail)
        m.set_rhs_host(b_host)
        m.residual_norm()
        barrier()
        torch.cuda.synchronize()
        # Pipelined through the public API: the upload of step s+1's b (copy stream) overlaps
        # step s's V-cycle; the host blocks once per step on the 8-byte norm read-back.  Timed on
        # the host clock from before the first upload to the last norm's return (every H2D, every
        # V-cycle and every D2H inside), max over ranks.
        t0 = time.perf_counter()
        m.set_rhs_host(b_host)              # H2D of step 0's input + brick conversion (+ b ghost exchange)
        for st in range(ke):
            m.vcycle()
            m.residual_norm_async()         # norm + D2H of the step's result (8 bytes)
            if st + 1 < ke:
                m.set_rhs_host(b_host)      # next step's H2D, overlapping this V-cycle
            m.residual_norm_wait()
        te = max_over_ranks((time.perf_counter() - t0) * 1e3)
        e2e = {"value": world * n**3 * ke / (te / 1e3), "unit": "DOF/s", "h2d_bytes_per_step": int(b_host.numel() * 8),
               "d2h_bytes_per_step": 8, "steps": ke, "ms_per_step": te / ke}
        # (informational) the same metric over whole solves through mg_solve (Alg 1): one upload of b
        # per solve, V-cycles until max|b - Ax| < 1e-10 with the norm read back after every cycle,
        # then the solution x downloaded into pinned host memory (mg_get_solution_host)
        ks, cyc_tot = 3, 0
        x_host = torch.empty(m.shape, dtype=torch.float64, pin_memory=True)
        barrier()
        t0 = time.perf_counter()
        for _ in range(ks):
            m.set_rhs_host(b_host)
            m.set_solution(None)
            _, cyc, _ = m.solve(1e-10, 20)
            m.get_solution_host(x_host)
            cyc_tot += cyc
        ts = max_over_ranks((time.perf_counter() - t0) * 1e3)
        e2e["solve"] = {"value": world * n**3 * cyc_tot / (ts / 1e3), "unit": "DOF/s", "solves": ks,
                        "vcycles_per_solve": cyc_tot / ks, "ms_per_solve": ts / ks,
                        "h2d_bytes_per_solve": int(b_host.numel() * 8),
                        "d2h_bytes_per_solve": int(x_host.numel() * 8 + 8 * (cyc_tot / ks + 1))}

    launches = m.launches_per_vcycle()
    xbytes, xmsgs = m.exchange_stats()
    exchange = exchange_block(m, a, world, max_over_ranks, tm, ninst)
    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        cpu = cpu_baseline(a)
    if rank == 0:
        line = {
            "metric": METRIC, "value": dofs, "unit": "DOF/s", "n_gpus": world, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": t_ms / a.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": workload_name(a, pg), "n_local": [n, n, n], "proc_grid": list(pg),
                       "levels": a.levels, "smooths": [a.pre, a.post, a.bottom], "brick": a.brick_edge or 8,
                       "bc": {0: "periodic (paper)", 1: "dirichlet", 2: "neumann"}[a.bc],
                       "coefficients": "variable (smooth c)" if a.var_coef else "constant (paper)",
                       "fusion": "auto(full)" if not a.fusion else a.fusion,
                       "ca_period": a.ca_period or "auto", "ghost_mode": "all" if a.ghost_all else "auto",
                       "cuda_graph": not a.no_graph, "overlap": not a.no_overlap, "pdl": not a.no_pdl,
                       "transport": a.transport,
                       "coarse": {0: "auto", 1: "per-sweep launches", 2: "resident bottom", 3: "cluster solve",
                                  4: "grid solve"}[a.bottom_mode],
                       "bottom_solver": "conjugate gradients" if a.bottom_solver else "damped jacobi (paper)",
                       "temporal_blocking": {0: "off", 1: "one-brick CTA streams"}.get(
                           a.tb, "2x2-brick pencils, two-warp CTAs"),
                       "smoother": {1: "chebyshev", 2: "red-black gauss-seidel"}.get(a.smoother, "damped jacobi (paper)"),
                       "l2": "no flush: every level-0 field is 1 GiB > 126 MB L2 (inputs larger than L2)",
                       "parallelism": f"3D domain decomposition {pg[0]}x{pg[1]}x{pg[2]}"},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic,
                         "kernel": ("level-0 passes: %s (two sweeps per pass)" % pass_kernel if a.tb else
                                    "level-0 sweeps: sweep_col_kernel + interp-fused sweep_kernel"),
                         "passes_per_vcycle": npass0, "launch_ms": launch_ms,
                         "bytes_per_point_per_pass": bytes0 / pts / npass0,
                         "sweep_equivalent_gbs": sweep_equiv,
                         "peak_source": peak_src, "frac_of_8TBs": achieved / 8000.0},
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches * a.steps,
            "launches_per_step": launches,
            "clocks": clk,
            "final_residual_norm": norm,
            "exchange": dict(exchange, bytes_per_cycle_per_rank=xbytes, messages_per_cycle_per_rank=xmsgs),
            "levels": levels,
            "instrumented_ms_per_step": total_inst,
        }
        print(json.dumps(line), flush=True)
    m.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()

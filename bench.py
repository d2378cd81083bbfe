#!/usr/bin/env python
"""bench.py — fp64 Jacobi-PCG of the MAS implicit viscosity operator on B200.

Metric (BASELINE.json): "fp64 PCG iters/sec and HBM GB/s vs peak at 1/2/4/8
B200, 36M-cell grid".  Workload: config C3 — 3-component
viscosity, 256x256x512 = 33.5 M cells (the paper's 36 M-cell test problem,
PAPER.md P:748-758, is the shape model), synthetic coronal-like fields
(paper_conf_ipps_caplansl23_b200.workloads), tol 1e-12.

One step = one implicit viscosity step of the hot path: mas_op_update
(a2: copy kappa/c, Jacobi diagonal) + x := x0 + mas_pcg_solve (a3-a5) to
tol 1e-12.  value = PCG iterations / s over all ranks (strong scaling: the
same global grid for every N, r-slabs per rank).  Inputs (>= 268 MB per
field) exceed the 126 MB L2, so no explicit flush is needed.

Launch: python bench.py [--gpus N --steps K --warmup W]; N > 1 under
torch.distributed.run (one process per GPU, NCCL).  --impl reference times
the CPU oracle on the host cores (the only other place oracle/ runs).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_ipps_caplansl23_b200 import workloads as W  # noqa: E402

METRIC = "fp64 PCG iters/sec and HBM GB/s vs peak at 1/2/4/8 B200, 36M-cell grid"
UNIT = "PCG iters/s"
CONFIGS = {
    # name: (kind, nr, nt, np)
    "C3": ("viscosity", 256, 256, 512),
    # C4: weak scaling, (256 * N) x 256 x 512 on N GPUs (nr scaled below)
    "C4": ("viscosity", 256, 256, 512),
    # one rank's share of C3 at P = 8 (32 r-planes), to study the per-GPU
    # kernel efficiency that bounds 8-GPU strong scaling
    "C3s8": ("viscosity", 32, 256, 512),
    # the whole C4 problem of 8 GPUs (268 M cells) on one B200
    "C4x8": ("viscosity", 2048, 256, 512),
    "C2": ("conduction", 128, 128, 256),
    # C2 with field-aligned conduction: kernel A, the
    # L_par kernel and kernel B per iteration (one GPU)
    "C2a": ("aniso", 128, 128, 256),
    # C2's conduction step with the temperature on the theta NODES, pole rows
    # one value per radius: 128 x 129 x 256 unknowns
    "C2t": ("tnode", 128, 128, 256),
    "C1": ("mms", 16, 24, 32),
}
# algorithmic bytes per cell per iteration: kernel A reads
# r, p_old, x (ncomp each) + dinv, kappa, c and writes p, q, x (ncomp each);
# kernel B reads r, q (ncomp) + dinv and writes r (ncomp).
def alg_bytes_per_cell(ncomp):
    a = 8 * (3 * ncomp + 3 + 3 * ncomp)
    if ncomp == 1:
        # scalar operator: x is read and written by every second kernel A (the
        # two-iteration x update), which then also reads p_{k-2}; per launch on
        # average one double less and half a double more (72 -> 68 B)
        a += -8 + 4
    b = 8 * (2 * ncomp + 1 + ncomp)
    return a, b


# single-reduction PCG (NEXT-1, --solver cg1): one kernel per iteration reads
# r, w, s, p, x (ncomp each) + dinv, kappa, c and writes s, r, p, x, w
def cg1_bytes_per_cell(ncomp):
    return 8 * (5 * ncomp + 3 + 5 * ncomp)


# the L_par kernel (NEXT-4, scalar): reads p_k and the 3 corner coefficients,
# reads and writes q
ANISO_BYTES_PER_CELL = 8 * (1 + 3 + 2)


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d.get("hbm_gbs", 6650.0)), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, smax, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 8:
                continue
            try:
                sm.append(float(parts[0]))
                smax = float(parts[1])
            except ValueError:
                continue
            for nm, v in zip(names, parts[4:8]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": smax,
                "reasons": sorted(reasons), "samples": len(sm)}


def make_problem(cfg: str, world: int = 1):
    kind, nr, nt, np_ = CONFIGS[cfg]
    if cfg == "C4":
        nr *= world
    return W.make(kind, nr=nr, nt=nt, np_=np_)


def scaling_of(cfg: str) -> str:
    return "weak" if cfg == "C4" else "strong"


def cpu_model() -> str:
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        kv = dict(ln.split(":", 1) for ln in out.splitlines() if ":" in ln)
        return "; ".join(f"{k.strip()}: {kv[k].strip()}" for k in
                         ("Model name", "Socket(s)", "Core(s) per socket", "Thread(s) per core")
                         if k in kv)
    except Exception:
        return "unknown"


def cpu_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def oracle_sample(prob, iters: int, threads: int):
    """Time the oracle (as it stands) on a bounded sample: `iters` fixed PCG
    iterations (tol = 0) on the full grid, minus a 1-iteration run to remove
    the setup (diagonal, initial residual).  Returns iters/s."""
    import oracle
    o = oracle.Oracle.for_problem(prob, threads)
    run = oracle_runner(o, prob, oracle_rhs(o, prob))
    # each oracle call allocates (and page-faults) its work vectors: at C3 that
    # is ~4 GB per call, as slow as several iterations, so the setup is
    # subtracted over two repetitions of run(1) / run(1 + iters)
    run(1)  # first touch
    t_short = t_long = 0.0
    for _ in range(2):
        t0 = time.perf_counter()
        run(1)
        t1 = time.perf_counter()
        run(1 + iters)
        t2 = time.perf_counter()
        t_short += t1 - t0
        t_long += t2 - t1
    dt = (t_long - t_short) / 2
    if not dt > 0.05 * t_long / 2:  # noise above the iterations' cost: keep the setup in
        dt = t_long / 2 * iters / (1 + iters)
    per_iter = dt / iters
    return 1.0 / per_iter, per_iter


def oracle_rhs(o, prob):
    if prob.extra.get("placement") == "theta-node":
        return o.tn_dirichlet_rhs(prob.kappa, prob.f, prob.ub_inner, prob.ub_outer)
    return o.dirichlet_rhs(prob.kappa, prob.f, prob.ub_inner, prob.ub_outer)


def oracle_runner(o, prob, f):
    """k fixed oracle PCG iterations (tol = 0) on the problem's operator."""
    if prob.extra.get("placement") == "theta-node":
        return lambda k: o.tn_pcg(prob.kappa, prob.c, f, prob.x0, 0.0, k)
    if prob.kpar is not None:
        return lambda k: o.pcg_aniso(prob.kappa, prob.c, prob.kpar, prob.bhat, f, prob.x0, 0.0, k)
    return lambda k: o.pcg(prob.kappa, prob.c, f, prob.x0, 0.0, k)


def host_dram_gbs(threads: int):
    """Host DRAM bandwidth (tools/hostbw.c, OpenMP, 2 GiB per array), the CPU
    roofline the oracle's time is set against: max of a copy
    counted with its write-allocate traffic (24 B/element) and a read-only
    sum (8 B/element).  Returns (max, copy, read) in GB/s."""
    import ctypes
    src = os.path.join(ROOT, "tools", "hostbw.c")
    so = os.path.join(ROOT, "tools", "libhostbw.so")
    try:
        if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
            subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-o", so, src])
        lib = ctypes.CDLL(so)
        for fn in (lib.host_copy_gbs, lib.host_read_gbs):
            fn.restype = ctypes.c_double
            fn.argtypes = [ctypes.c_longlong, ctypes.c_int]
        lib.host_set_threads.argtypes = [ctypes.c_int]
        lib.host_set_threads(int(threads))  # the oracle's 1-thread sample shares the OpenMP runtime
        cp = float(lib.host_copy_gbs(1 << 28, 3))
        rd = float(lib.host_read_gbs(1 << 28, 3))
        return max(cp, rd), cp, rd
    except Exception:
        return None, None, None


# bytes per cell per iteration of the oracle's textbook (unfused) PCG, per
# component: L p reads p, writes q (kappa, c shared: 2); <p,q> 2; x += a p,
# r -= a q 6; ||r|| 1; z = r / D 3; <r,z> 2; p = z + b p 3 -> 19 passes
# (SURVEY §8(d) counts 22 for the scalar case).
def oracle_bytes_per_cell(ncomp):
    return 8 * (2 + 19 * ncomp)


def run_reference(args):
    """--impl reference: the CPU oracle on this box's host cores, same config,
    metric and unit.  Each step is a bounded sample of the workload: 2 fixed
    oracle PCG iterations on the full grid, timed as run(1 + 2) - run(1) so
    the oracle's per-solve setup (diagonal, initial residual) is subtracted,
    as in the cpu_baseline leg."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    oracle.build()
    prob = make_problem(args.config)
    cores = cpu_cores()
    o = oracle.Oracle.for_problem(prob, cores)
    f = oracle_rhs(o, prob)
    per_step_iters = 2
    run = oracle_runner(o, prob, f)
    for _ in range(max(1, args.warmup)):
        run(1)
    t_short = t_long = 0.0
    for _ in range(args.steps):
        t0 = time.perf_counter()
        run(1)
        t1 = time.perf_counter()
        run(1 + per_step_iters)
        t2 = time.perf_counter()
        t_short += t1 - t0
        t_long += t2 - t1
    dt = t_long - t_short
    how = f"timed as run(1+{per_step_iters}) - run(1) (setup subtracted)"
    if not dt > 0.05 * t_long:  # timing noise above the iterations' cost: keep the setup in
        dt = t_long * per_step_iters / (1 + per_step_iters)
        how = f"timed as run(1+{per_step_iters}) scaled by {per_step_iters}/{1 + per_step_iters} (setup kept)"
    value = args.steps * per_step_iters / dt
    sample = (f"{args.config} full grid {prob.shape}, ncomp {prob.ncomp}: {per_step_iters} fixed "
              f"oracle PCG iterations per step, {how}")
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * dt / args.steps,
            "higher_is_better": True, "scaling": scaling_of(args.config), "vs_baseline": None,
            "dtype": "f64",
            "data": "synthetic", "impl": "reference",
            "config": {"workload": args.config, "grid": list(prob.shape), "ncomp": prob.ncomp},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def volumes(mesh, tnode=False):
    """V_P = rC^2 dr sin(tC) dt dp (the inner-product weight of R9), for the
    bench's own x comparison; theta nodes: sin(tF) (tC_j - tC_{j-1}) and the
    polar-cap measures 1 -+ cos at the pole rows (R29)."""
    dr, dt, dp = np.diff(mesh.rF), np.diff(mesh.tF), np.diff(mesh.pF)
    if tnode:
        tC, tF = mesh.tC, mesh.tF
        mt = np.empty(len(tF))
        mt[1:-1] = np.sin(tF[1:-1]) * np.diff(tC)
        mt[0], mt[-1] = 1.0 - np.cos(tC[0]), 1.0 + np.cos(tC[-1])
    else:
        mt = np.sin(mesh.tC) * dt
    return (mesh.rC ** 2 * dr)[:, None, None] * mt[None, :, None] * dp[None, None, :]


def reference_solve(M, prob, rank, dev, tol):
    """Rank 0: the same global problem on one GPU (no communicator)."""
    import torch
    g = M.Grid(prob.mesh)
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(dev)
    tn = prob.extra.get("placement") == "theta-node"
    o = M.Operator(g, prob.ncomp, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer,
                   placement=M.MAS_PLACE_THETA_NODE if tn else M.MAS_PLACE_CELL)
    if prob.kpar is not None:
        o.set_aniso(d(prob.kpar), d(prob.bhat))
    f = d(prob.f)
    if prob.ub_inner is not None or prob.ub_outer is not None:
        o.dirichlet_rhs(None if prob.ub_inner is None else d(prob.ub_inner),
                        None if prob.ub_outer is None else d(prob.ub_outer), f)
    x = d(prob.x0)
    st, it, rel, _ = o.solve(f, x, tol, 20000)
    xr = x.cpu().numpy()
    o.close()
    g.close()
    del x, f
    torch.cuda.empty_cache()
    return {"iters": it, "x": xr, "status": st}


def check_parity(M, op, prob, x0, rhs, ref, extent, rank, world, dev, tol, dist):
    """One solve on the multi-GPU op; gather x to rank 0 and compare with the
    P = 1 reference (iterations +-1, x <= 1e-10 relative L2_V)."""
    import torch
    x = x0.clone()
    st, it, rel, _ = op.solve(rhs, x, tol, 20000)
    ext = [None] * world
    dist.all_gather_object(ext, extent)
    n = max(e[1] * e[3] for e in ext) * prob.shape[2] * prob.ncomp
    buf = torch.zeros(n, device=dev, dtype=torch.float64)
    buf[: x.numel()] = x.reshape(-1)
    bufs = [torch.empty_like(buf) for _ in range(world)] if rank == 0 else None
    dist.gather(buf, bufs, dst=0)
    res = torch.zeros(3, device=dev, dtype=torch.float64)
    if rank == 0:
        xg = np.full((prob.ncomp,) + prob.shape, np.nan)
        for b, (i0, nl, j0, ntl) in zip(bufs, ext):
            blk = b[: prob.ncomp * nl * ntl * prob.shape[2]].cpu().numpy()
            xg[:, i0:i0 + nl, j0:j0 + ntl] = blk.reshape(prob.ncomp, nl, ntl, prob.shape[2])
        V = volumes(prob.mesh, prob.extra.get("placement") == "theta-node")[None]
        xr = ref["x"]
        err = float(np.sqrt((V * (xg - xr) ** 2).sum() / (V * xr ** 2).sum()))
        res[0], res[1], res[2] = err, ref["iters"], float(np.isnan(xg).any())
    dist.broadcast(res, src=0)
    err, it_ref, nan = float(res[0]), int(res[1]), bool(res[2])
    its = torch.tensor([it], device=dev, dtype=torch.float64)
    lo, hi = its.clone(), its.clone()
    dist.all_reduce(lo, op=dist.ReduceOp.MIN)
    dist.all_reduce(hi, op=dist.ReduceOp.MAX)
    ok = (st == M.MAS_OK and not nan and lo.item() == hi.item() and abs(it - it_ref) <= 1
          and err <= 1e-10)
    okt = torch.tensor([1.0 if ok else 0.0], device=dev, dtype=torch.float64)
    dist.all_reduce(okt, op=dist.ReduceOp.MIN)
    return {"ok": bool(okt.item() == 1.0), "iters": it, "iters_p1": it_ref, "x_rel_l2_V_vs_p1": err,
            "bound": "iters +-1, x <= 1e-10 (north_star)"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C3", choices=sorted(CONFIGS))
    ap.add_argument("--tol", type=float, default=1e-12)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-replay", action="store_true",
                    help="skip the kernel-replay timing (e.g. for an ncu launch list of the timed steps only)")
    ap.add_argument("--cpu-iters", type=int, default=6)
    ap.add_argument("--solver", default="pcg", choices=["pcg", "cg1"],
                    help="pcg: two fused kernels / two reductions per iteration; cg1: the "
                         "single-reduction (Chronopoulos-Gear) loop, one kernel per iteration "
                         "(NEXT-1, one GPU)")
    ap.add_argument("--ptheta", type=int, default=1,
                    help="(r, theta) decomposition: theta bands per r-slab (must divide --gpus)")
    ap.add_argument("--transport", default="auto", choices=["auto", "p2p", "nccl"],
                    help="multi-GPU PCG loop: P2P (NVLink peer memory: mailbox allreduce + "
                         "in-place seam reads, one CUDA graph per rank) or NCCL; auto = P2P "
                         "if every rank can map its peers, else NCCL")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    from paper_conf_ipps_caplansl23_b200 import build as B
    if rank == 0:
        B.build()
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
        dist.barrier()
    from paper_conf_ipps_caplansl23_b200 import maspcg as M

    prob = make_problem(args.config, world)
    nr, nt, np_ = prob.shape
    distinfo = None
    if world > 1:
        obj = [M.mas_comm_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        distinfo = (world, rank, obj[0])
    grid = M.Grid(prob.mesh, distinfo, ptheta=args.ptheta if world > 1 else 1)
    i0, nl, j0, ntl = grid.i0, grid.nl, grid.j0, grid.ntl
    tnode = prob.extra.get("placement") == "theta-node"
    if tnode:  # theta nodes: nt + 1 rows (r-slabs only)
        if args.ptheta != 1:
            raise SystemExit("C2t (theta-node placement) needs r-slabs (--ptheta 1)")
        nt, j0, ntl = nt + 1, 0, nt + 1
    sl = (slice(i0, i0 + nl), slice(j0, j0 + ntl))
    slc = (slice(None),) + sl
    nc = prob.ncomp

    def to_dev(a):
        return torch.from_numpy(np.ascontiguousarray(a)).to(dev)

    kappa = to_dev(prob.kappa[sl])
    cmass = to_dev(prob.c[sl])
    f = to_dev(prob.f[slc])
    x0 = to_dev(prob.x0[slc])
    x = x0.clone()
    aniso = prob.kpar is not None
    if aniso:  # NEXT-4 (r-slabs; either transport)
        if args.ptheta != 1:
            raise SystemExit("C2a (field-aligned conduction) needs r-slabs (--ptheta 1)")
        kpar = to_dev(prob.kpar[sl])
        bhat = to_dev(prob.bhat[(slice(None),) + sl])

    def make_op(use_p2p):
        o = M.Operator(grid, nc, kappa, cmass, prob.bc_inner, prob.bc_outer,
                       placement=M.MAS_PLACE_THETA_NODE if tnode else M.MAS_PLACE_CELL)
        if aniso:
            o.set_aniso(kpar, bhat)
        if args.solver == "cg1":
            o.set_single_reduction(True)
        tr = "single-gpu"
        if world > 1:
            tr = "nccl"
            if use_p2p:
                try:
                    o.enable_p2p()
                    tr = "p2p"
                except M.MasError as e:  # collective verdict: every rank keeps NCCL
                    if args.transport == "p2p":
                        raise
                    tr = f"nccl (p2p unavailable: {e})"
        return o, tr

    op, transport = make_op(args.transport != "nccl")
    ubi = to_dev(prob.ub_inner[:, j0:j0 + ntl]) if prob.ub_inner is not None else None
    ubo = to_dev(prob.ub_outer[:, j0:j0 + ntl]) if prob.ub_outer is not None else None
    rhs = f.clone()
    if ubi is not None or ubo is not None:
        op.dirichlet_rhs(ubi, ubo, rhs)

    # N > 1: self-check before timing.  Rank 0 solves the same global problem
    # on its own GPU (P = 1); every rank's slab of x is gathered and compared
    # (north_star: iterations +-1, x <= 1e-10 relative L2_V).  If the P2P
    # transport fails the check, the op falls back to NCCL and is re-checked.
    parity = None
    if world > 1:
        ref = reference_solve(M, prob, rank, dev, args.tol) if rank == 0 else None
        parity = check_parity(M, op, prob, x0, rhs, ref, (i0, nl, j0, ntl), rank, world, dev,
                              args.tol, dist)
        if not parity["ok"] and transport == "p2p" and args.transport == "auto":
            op.close()
            op, transport = make_op(False)
            parity = check_parity(M, op, prob, x0, rhs, ref, (i0, nl, j0, ntl), rank, world, dev,
                                  args.tol, dist)
            parity["fallback"] = "p2p failed the P=1 check; NCCL transport used"
        if not parity["ok"]:
            raise SystemExit(f"multi-GPU result differs from the P=1 solve: {parity}")
    stream = torch.cuda.current_stream()
    maxit = 20000

    def step(prof=False):
        op.update(kappa, cmass)           # a2: coefficients + Jacobi diagonal (1 kernel)
        if aniso:                         # NEXT-4: corner coefficients + their diagonal
            op.set_aniso(kpar, bhat)
        x.copy_(x0)                       # warm start x0 = v^n (R12)
        st, it, rel, _ = op.solve(rhs, x, args.tol, maxit)
        if st != M.MAS_OK:
            raise RuntimeError(f"solve status {st}")
        return it, op.launch_count + 1

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    # timed region: the production path (one GPU, or multi-GPU with the P2P
    # transport: the whole PCG loop is one CUDA graph per rank with a
    # device-side while node; multi-GPU NCCL: host-driven loop with NCCL
    # between the kernels)
    clocks = ClockSampler(local)
    clocks.start()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    e0.record(stream)
    iters_total, launches = 0, 0
    for _ in range(args.steps):
        it, nlaunch = step()
        iters_total += it
        launches += nlaunch
    e1.record(stream)
    torch.cuda.synchronize()
    clk = clocks.stop()
    t_ms = e0.elapsed_time(e1)
    if world > 1:
        tt = torch.tensor([t_ms], device=dev, dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_ms = float(tt.item())
        dist.barrier()
    # the same K steps again with every kernel A / kernel B launch bracketed by
    # CUDA events on the solve stream (host-driven loop): per-kernel durations
    op.set_profiling(True)
    ka, kb, kc = [], [], []
    e2, e3 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e2.record(stream)
    for _ in range(args.steps):
        step()
        a_ms, b_ms, n = op.kernel_times()
        ka.append(a_ms)
        kb.append(b_ms)
        kc.append(op.aniso_time())
    e3.record(stream)
    torch.cuda.synchronize()
    op.set_profiling(False)
    t_prof_ms = e2.elapsed_time(e3)
    # device time per launch of the iteration kernels from back-to-back CUDA
    # graph replays (no host dispatch between launches; mas_op_kernel_bench)
    replay = None
    if world == 1 and not args.no_replay:
        ra, rb, rc = op.kernel_bench(20)
        replay = {"A_ms": ra, "B_ms": rb or None, "Lpar_ms": rc or None,
                  "note": "20 launches of each kernel in a CUDA graph on the op's stream, each "
                          "after an L2 flush (a read sweep over 2x L2) and a PCG-state reset; the same graph without "
                          "the kernels is subtracted (CUDA events; device time, cold L2); the op's "
                          "vectors hold test values"}
    comm = None
    if world > 1:  # the exchange steps of the NCCL loop, measured on this op (collective)
        seam_us, ar_us, seam_b = op.comm_bench(20)
        mx = torch.tensor([seam_us, ar_us, seam_b], device=dev, dtype=torch.float64)
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        seam_us, ar_us, seam_b = (float(v) for v in mx.tolist())
        comm = {"seam_bytes_per_iter_max_rank": seam_b, "seam_us": seam_us,
                "seam_GBs": seam_b / (seam_us * 1e3) if seam_us > 0 else None,
                "seam_frac_of_nvlink_900GBs": (seam_b / (seam_us * 1e3) / 900.0) if seam_us > 0 else None,
                "allreduce_2dbl_us": ar_us,
                "note": "NCCL grouped send/recv of the r and p edge planes and a 2-double "
                        "ncclAllReduce, max over ranks (mas_op_comm_bench); the P2P transport "
                        "reads the same planes in place inside kernel A"}
    iters_per_solve = iters_total / args.steps
    value = iters_total / (t_ms / 1e3)  # the solve is one global problem: iterations are shared

    # roofline of the dominant kernel (kernel A), algorithmic bytes / its
    # average CUDA-event duration over the timed region
    cells = nr * nt * np_
    cells_local = nl * ntl * np_
    a_b, b_b = alg_bytes_per_cell(nc)
    if args.solver == "cg1":  # one kernel per iteration (kernel_times' A), no kernel B
        a_b, b_b = cg1_bytes_per_cell(nc), 0
    c_b = ANISO_BYTES_PER_CELL if aniso else 0
    fused = aniso and op.aniso_fused
    if fused:  # L_par inside kernel A: + the corner coefficients (a, b, e) per cell
        a_b, c_b = a_b + 24, 0
    a_ms = statistics.mean(ka)
    b_ms = statistics.mean(kb)
    peak, peak_src = load_peaks()
    achieved = a_b * cells_local / (a_ms / 1e3) / 1e9
    c_ms = statistics.mean(kc)
    iter_gbs = (a_b + b_b + c_b) * cells / (t_ms / 1e3 / iters_total) / 1e9
    traffic = None
    # the dominant kernel by device time: kernel A, or on C2a the L_par kernel
    dom = ("k_aniso<PCGA> (L_par)", c_b, c_ms, "kaniso") if aniso and c_b and c_ms > a_ms else \
        ("k_stencil<PCGA> + fused L_par (kernel A)", a_b, a_ms, "kernelA_lpar") if fused else \
        ("k_stencil<CG1> (single-reduction iteration)", a_b, a_ms, "cg1") if args.solver == "cg1" else \
        ("k_stencil<PCGA> (kernel A)", a_b, a_ms, "kernelA")
    dom_achieved = dom[1] * cells_local / (dom[2] / 1e3) / 1e9
    prof_json = os.path.join(ROOT, "profiles", f"ncu_{args.config}_{dom[3]}.json")
    if os.path.exists(prof_json):
        with open(prof_json) as fh:
            traffic = json.load(fh).get("dram_bytes_per_launch")

    # e2e: the same step through the C ABI with HOST buffers (pinned): the
    # library stages kappa, c, rhs, x0 to the device and copies x back.
    e2e = None
    if not args.no_e2e:
        pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()
        hk, hc, hf, hx0 = pin(prob.kappa[sl]), pin(prob.c[sl]), rhs.cpu().pin_memory(), \
            pin(prob.x0[slc])
        ksteps = args.steps
        # the solve overwrites x in place: x0 is refilled into the pinned
        # buffer between steps, outside the timed intervals (a host memcpy the
        # caller does, not library work); one untimed warm-up step allocates
        # the library's host-staging buffers
        hx = hx0.clone().pin_memory()
        if aniso:
            hkp, hb = pin(prob.kpar[sl]), pin(prob.bhat[(slice(None),) + sl])
        op.update(hk, hc)
        if aniso:
            op.set_aniso(hkp, hb)
        op.solve(hf, hx, args.tol, maxit)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        te, e2e_iters = 0.0, 0
        h0, h1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        for sidx in range(ksteps):
            hx.copy_(hx0)
            torch.cuda.synchronize()
            h0.record(stream)
            op.update(hk, hc)
            if aniso:
                op.set_aniso(hkp, hb)
            st, it, rel, _ = op.solve(hf, hx, args.tol, maxit)
            h1.record(stream)
            torch.cuda.synchronize()
            te += h0.elapsed_time(h1)
            e2e_iters += it
        if world > 1:
            tt = torch.tensor([te], device=dev, dtype=torch.float64)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            te = float(tt.item())
        h2d = (2 + 2 * nc + (4 if aniso else 0)) * cells_local * 8
        e2e = {"value": e2e_iters / (te / 1e3), "unit": UNIT, "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": nc * cells_local * 8,
               "note": "pinned host kappa, c, rhs, x0 (+ kpar, bhat for C2a) -> device inside the "
                       "timed region; x -> host; all K steps (per-step CUDA events, x0 refilled "
                       "between them); 1 untimed warm-up step"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cores = cpu_cores()
        v, per = oracle_sample(prob, args.cpu_iters, cores)
        # the survey's single-thread point (SURVEY §8(d) timing protocol: C1
        # and C2-sized grids), fixed iterations on the same grid
        hbw, hcp, hrd = host_dram_gbs(cores)
        v1 = per1 = None
        if cells <= 5_000_000:
            v1, per1 = oracle_sample(prob, 2, 1)
        ob = oracle_bytes_per_cell(nc) * cells * v / 1e9
        cpu = {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle",
               "host_dram_gbs": hbw, "host_copy_gbs_with_write_allocate": hcp,
               "host_read_gbs": hrd, "oracle_alg_gbs": ob,
               # below ~256 MB per iteration the oracle's vectors live in the host caches
               # and a DRAM fraction means nothing (C1)
               "oracle_frac_of_host_dram": (ob / hbw) if hbw and
               oracle_bytes_per_cell(nc) * cells >= 256e6 else None,
               "cpu_model": cpu_model(),
               "one_thread": None if v1 is None else {
                   "value": v1, "unit": UNIT, "cores": 1,
                   "sample": f"{args.config} full grid, 2 fixed oracle PCG iterations, setup "
                             f"subtracted; {per1:.3f} s/iteration"},
               "sample": f"{args.config} full grid, {args.cpu_iters} fixed oracle PCG iterations, "
                         f"setup subtracted via 1-iteration runs (2 repetitions); {per:.3f} s/iteration"}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": t_ms / args.steps,
            "higher_is_better": True, "scaling": scaling_of(args.config), "vs_baseline": None,
            "dtype": "f64", "data": "synthetic",
            "config": {"workload": args.config, "grid": [nr, nt, np_], "ncomp": nc,
                       "cells": cells, "tol": args.tol, "iters_per_solve": iters_per_solve,
                       "parallelism": (f"r-slab x{world}" if args.ptheta == 1 or world == 1 else
                                       f"(r,theta) {world // args.ptheta}x{args.ptheta}"),
                       "transport": transport,
                       "solver": args.solver,
                       **({"lpar": "fused into kernel A" if fused else "separate k_aniso kernel"}
                          if aniso else {}),
                       "l2": (f"no flush: one iteration streams {(a_b + b_b + c_b) * cells_local / 1e6:.0f}"
                              f" MB ({8 * cells_local / 1e6:.0f} MB per field) through the 126 MB L2"),
                       "step": "mas_op_update + " + ("mas_op_set_aniso + " if aniso else "") +
                               "x:=x0 + mas_pcg_solve"},
            "roofline": {"bound": "hbm", "kernel": dom[0],
                         "achieved": dom_achieved, "peak": peak, "unit": "GB/s",
                         "frac": dom_achieved / peak, "traffic": traffic,
                         "alg_bytes_per_cell": dom[1], "avg_ms": dom[2], "peak_source": peak_src},
            "kernels": {"A_ms": a_ms, "B_ms": b_ms,
                        "timing": "per-launch CUDA events in a second pass of the same K steps "
                                  "(host-driven loop); value is the graph-mode pass",
                        "profiled_pass_ms_per_step": t_prof_ms / args.steps,
                        "A_GBs": achieved,
                        **({"Lpar_ms": c_ms, "Lpar_GBs": c_b * cells_local / (c_ms / 1e3) / 1e9,
                            "Lpar_alg_bytes_per_cell": c_b} if aniso and c_ms > 0 else {}),
                        "B_GBs": b_b * cells_local / (b_ms / 1e3) / 1e9 if b_ms > 0 else None,
                        "iter_alg_GBs": iter_gbs, "iter_frac": iter_gbs / peak,
                        "alg_bytes_per_cell_iter": a_b + b_b + c_b,
                        **({"replay": {**replay,
                                       "A_frac": a_b * cells_local / (replay["A_ms"] / 1e3) / 1e9 / peak,
                                       "B_frac": (b_b * cells_local / (replay["B_ms"] / 1e3) / 1e9 / peak)
                                       if replay["B_ms"] else None,
                                       "Lpar_frac": (c_b * cells_local / (replay["Lpar_ms"] / 1e3) / 1e9 / peak)
                                       if replay["Lpar_ms"] else None}} if replay else {})},
            "e2e": e2e,
            **({"parity": parity, "comm": comm} if world > 1 else {}),
            "gpu_launches": launches,
            "clocks": clk,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())

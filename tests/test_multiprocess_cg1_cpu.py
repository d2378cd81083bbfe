"""World-size-2 `gloo` test on CPU of the single-reduction (NEXT-1) r-slab
protocol the library's NCCL loop uses (capi.cpp cg1_solve):
per iteration the seams of r, w = L D^-1 r and s, and ONE allreduce of the
three rank-local sums (gamma, delta, ||r||^2); every rank then takes the
stop / alpha / beta decision from identical global values.  The slab
arithmetic is the oracle's (mas_ref_op_apply_slab, mas_ref_dot_slab, pinned
bitwise to the monolithic operator); the recurrence is the oracle's CG1
(R28).  Result: iterations +-1 and x <= 1e-10 against the monolithic
mas_ref_pcg_solve_cg1, and exactly one allreduce per iteration."""
import math
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from test_multiprocess_cpu import free_port, seam_exchange

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import sys
    sys.path.insert(0, ROOT)
    import oracle
    from paper_conf_ipps_caplansl23_b200 import maspcg as M
    from paper_conf_ipps_caplansl23_b200 import workloads as W
    try:
        prob = W.viscosity_problem(9, 8, 16, warm=False)
        prob.kappa = prob.kappa * 40.0
        nr, nt, np_ = prob.shape
        i0, nl = M.mas_partition(nr, world, rank)
        o = oracle.Oracle.for_problem(prob)
        kext = torch.zeros((1, nl + 2, nt, np_), dtype=torch.float64)
        kext[0, 1:nl + 1] = torch.from_numpy(prob.kappa[i0:i0 + nl])
        seam_exchange(kext, nl, rank, world)
        c = prob.c[i0:i0 + nl]
        D = o.diag(prob.kappa, prob.c)[i0:i0 + nl][None]
        f = prob.f[:, i0:i0 + nl]
        nallred = [0]

        def allsum3(a, b, cc):
            nallred[0] += 1
            t = torch.tensor([a, b, cc], dtype=torch.float64)
            dist.all_reduce(t)
            return [float(v) for v in t]

        def Lslab(u):
            ext = torch.zeros((3, nl + 2, nt, np_), dtype=torch.float64)
            ext[:, 1:nl + 1] = torch.from_numpy(u)
            seam_exchange(ext, nl, rank, world)
            return o.apply_slab(i0, nl, kext[0].numpy(), c, ext.numpy())

        dl = lambda a, b: o.dot_slab(i0, nl, a, b)
        x = np.zeros_like(f)
        r = f.copy()                          # x0 = 0
        ff = allsum3(dl(f, f), 0.0, 0.0)[0]
        u = r / D
        w = Lslab(u)
        gam, dlt, rr = allsum3(dl(r, u), dl(w, u), dl(r, r))
        alpha, beta = gam / dlt, 0.0
        p, s = u.copy(), w.copy()
        it = 0
        for k in range(1, 500):
            x += alpha * p
            r -= alpha * s
            u = r / D
            w = Lslab(u)
            g_new, dlt, rr = allsum3(dl(r, u), dl(w, u), dl(r, r))   # the ONE allreduce
            if math.sqrt(rr) <= prob.tol * math.sqrt(ff):
                it = k
                break
            beta = g_new / gam
            alpha = g_new / (dlt - beta * g_new / alpha)
            gam = g_new
            p = u + beta * p
            s = w + beta * s
        xall = [None] * world
        dist.all_gather_object(xall, (i0, x, it, nallred[0]))
        out = {}
        if rank == 0:
            xfull = np.concatenate([b for _, b, _, _ in sorted(xall, key=lambda t: t[0])], axis=1)
            rc, xo, ito, _, _ = o.pcg_cg1(prob.kappa, prob.c, prob.f, np.zeros_like(prob.f), prob.tol, 500)
            V = o.volumes()[None]
            out = {"it": it, "ito": ito, "err": math.sqrt((V * (xfull - xo) ** 2).sum() / (V * xo ** 2).sum()),
                   "allreduces": [n for _, _, _, n in xall], "its": [t for _, _, t, _ in xall]}
        q.put((rank, out))
    except Exception as e:  # surface errors to the parent
        q.put((rank, {"error": repr(e)}))
    finally:
        dist.destroy_process_group()


def test_gloo_single_reduction_protocol():
    import oracle
    oracle.build()
    from paper_conf_ipps_caplansl23_b200 import build as B
    B.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
    for r in range(2):
        assert "error" not in res[r], res[r]
    out = res[0]
    assert len(set(out["its"])) == 1
    assert abs(out["it"] - out["ito"]) <= 1 and out["err"] <= 1e-10, out
    # <f,f> once, the init once, then exactly one allreduce per iteration
    assert out["allreduces"] == [2 + out["it"]] * 2, out["allreduces"]

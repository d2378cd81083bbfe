"""CPU tests of the r-slab protocol of the field-aligned conduction term
(NEXT-4; DESIGN.md §5.3 "Multi-rank"), the host logic the CUDA driver
implements:

* a rank owning planes [i0, i0+nl) needs the ghost planes i0-1 / i0+nl of the
  field and the corner plane i0+nl of (kpar, b), which is rank+1's first
  plane; with them the slab-local L_par equals the monolithic one BITWISE
  (oracle mas_ref_aniso_apply_slab vs mas_ref_aniso_apply, P = 1..4);
* world-size-2 `gloo`: the same exchanges as real inter-process traffic, then
  a distributed Jacobi-PCG on L_iso + L_par (rank-local sigma partials summed
  by an allreduce) matches the monolithic oracle PCG (+-1 iteration, 1e-10).
"""
import math
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_caplansl23_b200 import workloads as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def slab_inputs(prob, x, i0, nl):
    nr, nt, np_ = prob.shape
    ncomp = x.shape[0]
    xe = np.zeros((ncomp, nl + 2, nt, np_))
    xe[:, 1:nl + 1] = x[:, i0:i0 + nl]
    if i0 > 0:
        xe[:, 0] = x[:, i0 - 1]
    if i0 + nl < nr:
        xe[:, nl + 1] = x[:, i0 + nl]
    ke = np.zeros((nl + 1, nt, np_))
    be = np.zeros((3, nl + 1, nt, np_))
    top = min(i0 + nl + 1, nr)
    ke[:top - i0] = prob.kpar[i0:top]
    be[:, :top - i0] = prob.bhat[:, i0:top]
    return ke, be, xe


@pytest.mark.parametrize("P", [1, 2, 3, 4])
def test_aniso_slab_apply_bitwise(oracle_mod, P):
    prob = W.aniso_conduction_problem(11, 12, 16)
    o = oracle_mod.Oracle.for_problem(prob)
    x = W.random_field((2,) + prob.shape, 3)
    ymono = o.aniso_apply(prob.kpar, prob.bhat, x)
    parts = []
    for rank in range(P):
        i0, nl = oracle_mod.partition(prob.shape[0], P, rank)
        ke, be, xe = slab_inputs(prob, x, i0, nl)
        parts.append(o.aniso_apply_slab(i0, nl, ke, be, xe))
    assert np.array_equal(np.concatenate(parts, axis=1), ymono)


def test_aniso_slab_needs_the_corner_plane_above(oracle_mod):
    """Dropping the neighbour's corner plane (zeros instead) changes the
    last plane of the slab: the exchange is load-bearing."""
    prob = W.aniso_conduction_problem(8, 8, 16)
    o = oracle_mod.Oracle.for_problem(prob)
    x = W.random_field((1,) + prob.shape, 4)
    i0, nl = oracle_mod.partition(8, 2, 0)
    ke, be, xe = slab_inputs(prob, x, i0, nl)
    good = o.aniso_apply_slab(i0, nl, ke, be, xe)
    ke[nl] = 0.0
    bad = o.aniso_apply_slab(i0, nl, ke, be, xe)
    assert np.array_equal(good[:, :nl - 1], bad[:, :nl - 1])
    assert not np.array_equal(good[:, nl - 1], bad[:, nl - 1])


# ---------------------------------------------------------------------------
# world-size-2 gloo
# ---------------------------------------------------------------------------
def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def exchange_planes(ext, nl, rank, world, lo=True, hi=True):
    """ext [c, nl+2, ...]: send planes 1 / nl to rank-1 / rank+1, receive the
    neighbours' edge planes into 0 / nl+1."""
    reqs, rl, rh = [], None, None
    if rank > 0:
        reqs.append(dist.isend(ext[:, 1].contiguous(), rank - 1))
        rl = torch.empty_like(ext[:, 0])
        reqs.append(dist.irecv(rl, rank - 1))
    if rank < world - 1:
        reqs.append(dist.isend(ext[:, nl].contiguous(), rank + 1))
        rh = torch.empty_like(ext[:, 0])
        reqs.append(dist.irecv(rh, rank + 1))
    for r in reqs:
        r.wait()
    if rl is not None and lo:
        ext[:, 0] = rl
    if rh is not None and hi:
        ext[:, nl + 1] = rh


def allsum(v):
    t = torch.tensor([v], dtype=torch.float64)
    dist.all_reduce(t)
    return float(t.item())


def worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import sys
    sys.path.insert(0, ROOT)
    import oracle
    out = {}
    try:
        prob = W.aniso_conduction_problem(10, 8, 16)
        nr, nt, np_ = prob.shape
        i0, nl = oracle.partition(nr, world, rank)
        o = oracle.Oracle.for_problem(prob)
        # static exchanges: kappa ghosts (L_iso) and the corner plane above (L_par)
        kext = torch.zeros((1, nl + 2, nt, np_), dtype=torch.float64)
        kext[0, 1:nl + 1] = torch.from_numpy(prob.kappa[i0:i0 + nl])
        exchange_planes(kext, nl, rank, world)
        cext = torch.zeros((4, nl + 2, nt, np_), dtype=torch.float64)  # kpar, b_r, b_t, b_p
        cext[0, 1:nl + 1] = torch.from_numpy(prob.kpar[i0:i0 + nl])
        cext[1:, 1:nl + 1] = torch.from_numpy(prob.bhat[:, i0:i0 + nl])
        exchange_planes(cext, nl, rank, world, lo=False)
        ke = cext[0, 1:].numpy().copy()
        be = cext[1:, 1:].numpy().copy()
        c = prob.c[i0:i0 + nl]

        def L(pext):
            return (o.apply_slab(i0, nl, kext[0].numpy(), c, pext.numpy())
                    + o.aniso_apply_slab(i0, nl, ke, be, pext.numpy()))

        D = (o.diag(prob.kappa, prob.c) + o.aniso_diag(prob.kpar, prob.bhat))[i0:i0 + nl]
        fg = o.dirichlet_rhs(prob.kappa, prob.f, prob.ub_inner, prob.ub_outer)
        f = fg[:, i0:i0 + nl]
        dot = lambda a, b: allsum(o.dot_slab(i0, nl, a, b))
        bn = math.sqrt(dot(f, f))
        xext = torch.zeros((1, nl + 2, nt, np_), dtype=torch.float64)
        xext[:, 1:nl + 1] = torch.from_numpy(prob.x0[:, i0:i0 + nl])
        exchange_planes(xext, nl, rank, world)
        xs = prob.x0[:, i0:i0 + nl].copy()
        r = f - L(xext)
        z = r / D[None]
        pext = torch.zeros((1, nl + 2, nt, np_), dtype=torch.float64)
        pext[:, 1:nl + 1] = torch.from_numpy(z)
        rho = dot(r, z)
        it = 0
        for k in range(1, 2000):
            exchange_planes(pext, nl, rank, world)
            qv = L(pext)
            p = pext[:, 1:nl + 1].numpy().copy()
            alpha = rho / dot(p, qv)
            xs += alpha * p
            r -= alpha * qv
            if math.sqrt(dot(r, r)) <= prob.tol * bn:
                it = k
                break
            z = r / D[None]
            rn = dot(r, z)
            pext[:, 1:nl + 1] = torch.from_numpy(z + (rn / rho) * p)
            rho = rn
        xall = [None] * world
        dist.all_gather_object(xall, (i0, xs, it))
        if rank == 0:
            xfull = np.concatenate([b for _, b, _ in sorted(xall, key=lambda t: t[0])], axis=1)
            rc, xo, ito, _, _ = oracle.solve_problem(prob)
            V = o.volumes()[None]
            out["pcg"] = (it, ito, math.sqrt((V * (xfull - xo) ** 2).sum() / (V * xo ** 2).sum()))
        q.put((rank, out))
    except Exception as e:  # surface errors to the parent
        q.put((rank, {"error": repr(e)}))
    finally:
        dist.destroy_process_group()


def test_gloo_aniso_r_slab_pcg():
    import oracle
    oracle.build()
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert "error" not in res[r], res[r]
    it, ito, err = res[0]["pcg"]
    assert abs(it - ito) <= 1 and err <= 1e-10, (it, ito, err)

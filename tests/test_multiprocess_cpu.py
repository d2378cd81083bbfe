"""World-size-2 `gloo` tests on CPU of the multi-GPU (r-slab) path's host
logic, SURVEY.md §8(e):

* the library's partition (mas_partition) agrees across ranks and tiles nr;
* the NCCL unique id from rank 0 reaches every rank intact through
  torch.distributed (how bench.py bootstraps mas_dist_t);
* the seam protocol the CUDA driver uses (each rank sends its first plane to
  rank-1 and its last plane to rank+1, receives the neighbours' edge planes
  as ghost planes; dots are per-rank partials summed by an allreduce) turns
  slab-local operators into the monolithic one: matvec bitwise, PCG +-1
  iteration / 1e-10.  The slab arithmetic here is the oracle's
  (mas_ref_op_apply_slab); the exchange is real inter-process gloo traffic.
"""
import math
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def seam_exchange(x_ext, nl, rank, world):
    """x_ext: [ncomp, nl+2, nt, np] with interior planes 1..nl; fills ghosts."""
    reqs = []
    ncomp = x_ext.shape[0]
    recv_lo = torch.empty_like(x_ext[:, 0]) if rank > 0 else None
    recv_hi = torch.empty_like(x_ext[:, 0]) if rank < world - 1 else None
    if rank > 0:
        reqs.append(dist.isend(x_ext[:, 1].contiguous(), rank - 1))
        reqs.append(dist.irecv(recv_lo, rank - 1))
    if rank < world - 1:
        reqs.append(dist.isend(x_ext[:, nl].contiguous(), rank + 1))
        reqs.append(dist.irecv(recv_hi, rank + 1))
    for r in reqs:
        r.wait()
    if recv_lo is not None:
        x_ext[:, 0] = recv_lo
    if recv_hi is not None:
        x_ext[:, nl + 1] = recv_hi
    del ncomp


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
    from paper_conf_ipps_caplansl23_b200 import maspcg as M
    from paper_conf_ipps_caplansl23_b200 import workloads as W
    out = {}
    try:
        # 1. partition agreement
        for nr in (7, 256, 320):
            mine = M.mas_partition(nr, world, rank)
            allp = [None] * world
            dist.all_gather_object(allp, mine)
            out.setdefault("parts", []).append((nr, allp, oracle.partition(nr, world, rank)))
        # 2. NCCL unique id bootstrap (as bench.py does it)
        obj = [M.mas_comm_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        ids = [None] * world
        dist.all_gather_object(ids, obj[0])
        out["ids_equal"] = all(i == ids[0] for i in ids) and len(ids[0]) == 128
        # 3. seam protocol: distributed matvec and PCG with real exchanges
        prob = W.viscosity_problem(9, 8, 16, warm=False)
        prob.kappa = prob.kappa * 40.0
        nr, nt, np_ = prob.shape
        i0, nl = M.mas_partition(nr, world, rank)
        o = oracle.Oracle.for_problem(prob)
        x = W.random_field((3,) + prob.shape, 42)
        kext = torch.zeros((1, nl + 2, nt, np_), dtype=torch.float64)
        kext[0, 1:nl + 1] = torch.from_numpy(prob.kappa[i0:i0 + nl])
        seam_exchange(kext, nl, rank, world)
        xext = torch.zeros((3, nl + 2, nt, np_), dtype=torch.float64)
        xext[:, 1:nl + 1] = torch.from_numpy(x[:, i0:i0 + nl])
        seam_exchange(xext, nl, rank, world)
        c = prob.c[i0:i0 + nl]
        y = o.apply_slab(i0, nl, kext[0].numpy(), c, xext.numpy())
        yall = [None] * world
        dist.all_gather_object(yall, (i0, y))
        if rank == 0:
            yfull = np.concatenate([b for _, b in sorted(yall, key=lambda t: t[0])], axis=1)
            out["matvec_bitwise"] = bool(np.array_equal(yfull, o.apply(prob.kappa, prob.c, x)))
        # distributed Jacobi-PCG (textbook order) over the slabs
        D = o.diag(prob.kappa, prob.c)[i0:i0 + nl]
        f = prob.f[:, i0:i0 + nl]
        xs = np.zeros_like(f)
        dot = lambda a, b: allsum(o.dot_slab(i0, nl, a, b))
        bn = math.sqrt(dot(f, f))
        r = f.copy()  # x0 = 0
        z = r / D[None]
        pext = torch.zeros((3, nl + 2, nt, np_), dtype=torch.float64)
        pext[:, 1:nl + 1] = torch.from_numpy(z)
        rho = dot(r, z)
        it = 0
        for k in range(1, 500):
            seam_exchange(pext, nl, rank, world)
            qv = o.apply_slab(i0, nl, kext[0].numpy(), c, pext.numpy())
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
            rc, xo, ito, _, _ = o.pcg(prob.kappa, prob.c, prob.f, np.zeros_like(prob.f), prob.tol, 500)
            V = o.volumes()[None]
            out["pcg"] = (it, ito, math.sqrt((V * (xfull - xo) ** 2).sum() / (V * xo ** 2).sum()))
        q.put((rank, out))
    except Exception as e:  # surface errors to the parent
        q.put((rank, {"error": repr(e)}))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_r_slab_protocol(world):
    import oracle
    oracle.build()
    from paper_conf_ipps_caplansl23_b200 import build as B
    B.build()
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
    for nr, allp, orc in res[0]["parts"]:
        assert allp[0][0] == 0 and sum(n for _, n in allp) == nr
        for (a, n), (b, _) in zip(allp, allp[1:]):
            assert a + n == b
        assert tuple(allp[0]) == tuple(orc)
    assert res[0]["ids_equal"] and res[1]["ids_equal"]
    assert res[0]["matvec_bitwise"]
    it, ito, err = res[0]["pcg"]
    assert abs(it - ito) <= 1 and err <= 1e-10, (it, ito, err)


# ---------------------------------------------------------------------------
# (r, theta) decomposition (NEXT-3): ranks = pr x ptheta, theta fastest.  The
# r-seams go to rank -/+ ptheta, the theta-ghost rows (packed [comp][i][phi])
# to rank -/+ 1 within the r-slab, as in the library (capi.cpp tseams).
# ---------------------------------------------------------------------------
def block_exchange(ext, nl, ntl, rank, pr, pt):
    """ext: [ncomp, nl+2, ntl+2, np] with the block at [1:nl+1, 1:ntl+1]."""
    rr, rt = divmod(rank, pt)
    reqs, recv = [], {}

    def post(send, peer, key, like):
        reqs.append(dist.isend(send.contiguous(), peer))
        recv[key] = torch.empty_like(like)
        reqs.append(dist.irecv(recv[key], peer))

    inner = ext[:, :, 1:ntl + 1]
    if rr > 0:
        post(inner[:, 1], rank - pt, "rlo", inner[:, 0])
    if rr < pr - 1:
        post(inner[:, nl], rank + pt, "rhi", inner[:, 0])
    rows = ext[:, 1:nl + 1]
    if rt > 0:
        post(rows[:, :, 1], rank - 1, "tlo", rows[:, :, 0])
    if rt < pt - 1:
        post(rows[:, :, ntl], rank + 1, "thi", rows[:, :, 0])
    for q in reqs:
        q.wait()
    if "rlo" in recv:
        ext[:, 0, 1:ntl + 1] = recv["rlo"]
    if "rhi" in recv:
        ext[:, nl + 1, 1:ntl + 1] = recv["rhi"]
    if "tlo" in recv:
        ext[:, 1:nl + 1, 0] = recv["tlo"]
    if "thi" in recv:
        ext[:, 1:nl + 1, ntl + 1] = recv["thi"]


def worker_2d(rank, world, pt, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import sys
    sys.path.insert(0, ROOT)
    import oracle
    from paper_conf_ipps_caplansl23_b200 import maspcg as M
    from paper_conf_ipps_caplansl23_b200 import workloads as W
    out = {}
    try:
        pr = world // pt
        rr, rt = divmod(rank, pt)
        prob = W.viscosity_problem(6, 11, 16, warm=False)
        prob.kappa = prob.kappa * 40.0
        nr, nt, np_ = prob.shape
        i0, nl = M.mas_partition(nr, pr, rr)
        j0, ntl = M.mas_partition(nt, pt, rt)
        blk = (slice(i0, i0 + nl), slice(j0, j0 + ntl))
        o = oracle.Oracle.for_problem(prob)
        x = W.random_field((3,) + prob.shape, 42)

        def ext_of(a):  # a: [ncomp, nl, ntl, np] block -> exchanged ext
            e = torch.zeros((a.shape[0], nl + 2, ntl + 2, np_), dtype=torch.float64)
            e[:, 1:nl + 1, 1:ntl + 1] = torch.from_numpy(np.ascontiguousarray(a))
            block_exchange(e, nl, ntl, rank, pr, pt)
            return e.numpy()

        kext = ext_of(prob.kappa[None][(slice(None),) + blk])[0]
        c = prob.c[blk]
        y = o.apply_block(i0, nl, j0, ntl, kext, c, ext_of(x[(slice(None),) + blk]))
        yall = [None] * world
        dist.all_gather_object(yall, (i0, nl, j0, ntl, y))
        if rank == 0:
            yfull = np.full((3,) + prob.shape, np.nan)
            for a, n, b, m, yb in yall:
                yfull[:, a:a + n, b:b + m] = yb
            out["matvec_bitwise"] = bool(np.array_equal(yfull, o.apply(prob.kappa, prob.c, x)))
        # distributed Jacobi-PCG over the blocks (textbook order)
        D = o.diag(prob.kappa, prob.c)[blk]
        f = prob.f[(slice(None),) + blk]
        dot = lambda a, b: allsum(o.dot_block(i0, nl, j0, ntl, a, b))
        bn = math.sqrt(dot(f, f))
        xs = np.zeros_like(f)
        r = f.copy()
        p = r / D[None]
        rho = dot(r, p)
        it = 0
        for k in range(1, 500):
            qv = o.apply_block(i0, nl, j0, ntl, kext, c, ext_of(p))
            alpha = rho / dot(p, qv)
            xs += alpha * p
            r -= alpha * qv
            if math.sqrt(dot(r, r)) <= prob.tol * bn:
                it = k
                break
            z = r / D[None]
            rn = dot(r, z)
            p = z + (rn / rho) * p
            rho = rn
        xall = [None] * world
        dist.all_gather_object(xall, (i0, nl, j0, ntl, xs, it))
        if rank == 0:
            xfull = np.full((3,) + prob.shape, np.nan)
            for a, n, b, m, xb, _ in xall:
                xfull[:, a:a + n, b:b + m] = xb
            rc, xo, ito, _, _ = o.pcg(prob.kappa, prob.c, prob.f, np.zeros_like(prob.f), prob.tol, 500)
            V = o.volumes()[None]
            out["pcg"] = (it, ito, math.sqrt((V * (xfull - xo) ** 2).sum() / (V * xo ** 2).sum()),
                          {t[5] for t in xall})
        q.put((rank, out))
    except Exception as e:  # surface errors to the parent
        q.put((rank, {"error": repr(e)}))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,pt", [(2, 2), (4, 2)])
def test_gloo_r_theta_block_protocol(world, pt):
    import oracle
    oracle.build()
    from paper_conf_ipps_caplansl23_b200 import build as B
    B.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=worker_2d, args=(r, world, pt, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert "error" not in res[r], res[r]
    assert res[0]["matvec_bitwise"]
    it, ito, err, its = res[0]["pcg"]
    assert len(its) == 1 and abs(it - ito) <= 1 and err <= 1e-10, (it, ito, err, its)

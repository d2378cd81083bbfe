"""World-size-2 `gloo` test on CPU of bench.py's N > 1 self-check
(check_parity): every rank's slab of x is gathered to rank 0 and compared
with the P = 1 reference (iterations +-1, x <= 1e-10 relative L2_V); the
verdict must reach every rank.  The op is a stand-in whose solve writes the
reference slab (optionally perturbed on one rank, or with a skewed iteration
count), so the gather / slab placement / verdict logic is what is tested."""
import importlib.util
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as tmp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def load_bench():
    spec = importlib.util.spec_from_file_location("bench", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


class FakeM:
    MAS_OK = 0


class FakeOp:
    def __init__(self, xslab, iters):
        self.xslab, self.iters = xslab, iters

    def solve(self, rhs, x, tol, maxit):
        x.copy_(self.xslab)
        return 0, self.iters, 1e-13, None


def worker(rank, world, port, case, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import sys
        sys.path.insert(0, ROOT)
        from paper_conf_ipps_caplansl23_b200 import workloads as W
        b = load_bench()
        prob = W.viscosity_problem(9, 6, 8)
        rng = np.random.default_rng(3)
        xref = rng.standard_normal((prob.ncomp,) + prob.shape)
        nr = prob.shape[0]
        i0 = 0 if rank == 0 else nr // 2 + (nr % 2)
        nl = (nr // 2 + (nr % 2)) if rank == 0 else nr // 2
        xs = torch.from_numpy(np.ascontiguousarray(xref[:, i0:i0 + nl]))
        iters = 50
        if case == "perturbed" and rank == 1:
            xs = xs.clone()
            xs[0, 0, 0, 0] += 1e-6
        if case == "iters" and rank == 1:
            iters = 53
        ref = {"iters": 50, "x": xref} if rank == 0 else None
        res = b.check_parity(FakeM, FakeOp(xs, iters), prob, torch.zeros_like(xs), None, ref,
                             (i0, nl, 0, prob.shape[1]), rank, world, torch.device("cpu"), 1e-12, dist)
        q.put((rank, res["ok"], res["x_rel_l2_V_vs_p1"]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("case,expect", [("exact", True), ("perturbed", False), ("iters", False)])
def test_check_parity_gathers_slabs_and_agrees(case, expect):
    ctx = tmp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    ps = [ctx.Process(target=worker, args=(r, 2, port, case, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = [q.get(timeout=120) for _ in ps]
    for p in ps:
        p.join(60)
    assert all(ok == expect for _, ok, _ in out), out
    if case == "exact":
        assert all(err == 0.0 for _, _, err in out)

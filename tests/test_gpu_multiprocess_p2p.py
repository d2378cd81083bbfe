"""The P2P transport across real processes on ONE B200.

Two (or three) processes each own an r-slab of the same problem, as ranks of
a multi-GPU job would.  NCCL cannot place two ranks on one device, so the
setup-time collectives go through the library's "host exchange" test
transport (files in a shared directory, comm.cpp); everything on the solve
path is the multi-GPU code: cudaIpcGetMemHandle / cudaIpcOpenMemHandle of the
peers' r, p and mailbox buffers, kernel A reading the neighbour's edge planes
through the IPC mapping, the mailbox allreduce written by one process's kernel
and polled by the other's, and the per-rank CUDA-graph loop.  The processes'
kernels are time-sliced on the device, so each mailbox wait spans a context
switch (slow, but it must make progress and give the oracle's answer).
"""
import json
import math
import os
import subprocess
import sys

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import workloads as W

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
WORKER = r"""
import json, sys
import numpy as np, torch
sys.path.insert(0, {root!r})
from paper_conf_ipps_caplansl23_b200 import maspcg as M, workloads as W
P, rank, d, kind, nr, nt, np_, p2p, pt, cg1 = ({P}, int(sys.argv[1]), {d!r}, {kind!r}, {nr}, {nt}, {np_},
                                               {p2p}, {ptheta}, {cg1})
torch.cuda.set_device(0)
prob = W.make(kind, nr=nr, nt=nt, np_=np_, warm=False)
g = M.Grid(prob.mesh, dist=(P, rank, M.host_exchange_id(d)), ptheta=pt)
sl = (slice(g.i0, g.i0 + g.nl), slice(g.j0, g.j0 + g.ntl))
slc = (slice(None),) + sl
dv = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
op = M.Operator(g, prob.ncomp, dv(prob.kappa[sl]), dv(prob.c[sl]), prob.bc_inner, prob.bc_outer)
if cg1:  # the single-reduction loop first: enable_p2p then maps its buffers too
    op.set_single_reduction(True)
if p2p:
    op.enable_p2p()
if prob.kpar is not None:  # field-aligned conduction: neighbour p_k through the IPC mapping
    op.set_aniso(dv(prob.kpar[sl]), dv(prob.bhat[slc]))
f = dv(prob.f[slc])
op.dirichlet_rhs(dv(prob.ub_inner[:, g.j0:g.j0 + g.ntl]) if prob.ub_inner is not None else None,
                 None, f)
res = []
for _ in range(2):
    x = dv(prob.x0[slc])
    st, it, rel, hist = op.solve(f, x, prob.tol, prob.maxit, True)
    torch.cuda.synchronize()
    res.append((st, it))
np.save(f"{{d}}/x.{{rank}}.npy", x.cpu().numpy())
json.dump({{"res": res, "transport": op.transport, "i0": g.i0, "nl": g.nl, "j0": g.j0,
           "ntl": g.ntl, "hist": list(hist)}},
          open(f"{{d}}/out.{{rank}}.json", "w"))
op.close(); g.close()
"""


def run_procs(tmp_path, P, kind, shape, p2p=True, timeout=600, ptheta=1, cg1=False):
    d = str(tmp_path)
    src = WORKER.format(root=ROOT, P=P, d=d, kind=kind, nr=shape[0], nt=shape[1], np_=shape[2],
                        p2p=p2p, ptheta=ptheta, cg1=cg1)
    script = os.path.join(d, "worker.py")
    with open(script, "w") as fh:
        fh.write(src)
    procs = [subprocess.Popen([sys.executable, script, str(r)], stdout=subprocess.PIPE,
                              stderr=subprocess.STDOUT) for r in range(P)]
    outs = []
    for p in procs:
        try:
            o, _ = p.communicate(timeout=timeout)
        except subprocess.TimeoutExpired:
            for q in procs:
                q.kill()
            raise
        outs.append(o.decode(errors="replace"))
    for r, p in enumerate(procs):
        assert p.returncode == 0, f"rank {r}:\n{outs[r][-3000:]}"
    res = [json.load(open(os.path.join(d, f"out.{r}.json"))) for r in range(P)]
    xs = [np.load(os.path.join(d, f"x.{r}.npy")) for r in range(P)]
    return res, xs


@pytest.fixture(scope="module")
def built():
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    from paper_conf_ipps_caplansl23_b200 import build
    build.build()


@pytest.mark.parametrize("P,kind,shape,ptheta", [(2, "viscosity", (12, 16, 64), 1),
                                                 (3, "conduction", (13, 16, 32), 1),
                                                 (4, "viscosity", (10, 18, 64), 2),
                                                 (2, "aniso", (12, 16, 64), 1)])
def test_p2p_across_processes_matches_oracle(built, oracle_mod, tmp_path, P, kind, shape, ptheta):
    res, xs = run_procs(tmp_path, P, kind, shape, ptheta=ptheta)
    assert all(r["transport"] == "p2p" for r in res)
    prob = W.make(kind, nr=shape[0], nt=shape[1], np_=shape[2], warm=False)
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob)
    its = {tuple(map(tuple, r["res"])) for r in res}
    assert len(its) == 1, its  # every rank, both solves: same status and count
    (st1, it1), (st2, it2) = its.pop()
    assert st1 == st2 == 0 and it1 == it2 and abs(it1 - ito) <= 1
    V = oracle_mod.Oracle.for_problem(prob).volumes()[None]
    xg = np.full(xo.shape, np.nan)
    for r, xl in zip(res, xs):
        xg[:, r["i0"]:r["i0"] + r["nl"], r["j0"]:r["j0"] + r["ntl"]] = xl
    assert not np.isnan(xg).any()
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10


@pytest.mark.parametrize("P,kind,shape", [(2, "viscosity", (12, 16, 64)), (3, "conduction", (13, 16, 32))])
def test_single_reduction_p2p_across_processes(built, oracle_mod, tmp_path, P, kind, shape):
    """NEXT-1 over the P2P transport: each single-reduction kernel publishes its
    3 partial sums to every process's mailbox and the next kernel sums them
    there; the r, w, s halos come through the IPC mappings.  Against the
    oracle's CG1: +-2 iterations, x <= 1e-9 (SURVEY §8(f) NEXT-1 band)."""
    res, xs = run_procs(tmp_path, P, kind, shape, cg1=True)
    assert all(r["transport"] == "p2p" for r in res)
    prob = W.make(kind, nr=shape[0], nt=shape[1], np_=shape[2], warm=False)
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob, cg1=True)
    its = {tuple(map(tuple, r["res"])) for r in res}
    assert len(its) == 1, its
    (st1, it1), (st2, it2) = its.pop()
    assert st1 == st2 == 0 and it1 == it2 and abs(it1 - ito) <= 2
    V = oracle_mod.Oracle.for_problem(prob).volumes()[None]
    xg = np.full(xo.shape, np.nan)
    for r, xl in zip(res, xs):
        xg[:, r["i0"]:r["i0"] + r["nl"], r["j0"]:r["j0"] + r["ntl"]] = xl
    assert not np.isnan(xg).any()
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-9

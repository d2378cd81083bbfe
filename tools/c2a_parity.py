#!/usr/bin/env python
"""C2a at full size (128 x 128 x 256, field-aligned conduction, NEXT-4) solved
once as one rank and once as P ranks through the "virtual ranks" transport
(P host threads on one GPU: the r-slab multi-rank path with the corner-plane
seam at mas_op_set_aniso and the p_k seams after every kernel A).

Prints JSON: iterations per P (must agree within +-1) and the relative L2_V
difference of x (<= 1e-10)."""
import argparse
import json
import math
import os
os.environ.setdefault("MAS_TEST_TRANSPORTS", "1")  # virtual ranks (comm.cpp)
import sys
import threading

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_caplansl23_b200 import maspcg as M  # noqa: E402
from paper_conf_ipps_caplansl23_b200 import workloads as W  # noqa: E402


def solve(prob, P, key):
    res, errs = {}, []
    vid = M.virtual_ranks_id(key) if P > 1 else None

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            with torch.cuda.stream(torch.cuda.Stream()):
                g = M.Grid(prob.mesh, dist=(P, r, vid) if P > 1 else None)
                sl = slice(g.i0, g.i0 + g.nl)
                d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
                op = M.Operator(g, 1, d(prob.kappa[sl]), d(prob.c[sl]), prob.bc_inner, prob.bc_outer)
                op.set_aniso(d(prob.kpar[sl]), d(prob.bhat[:, sl]))
                f = d(prob.f[:, sl])
                op.dirichlet_rhs(d(prob.ub_inner), None, f)
                x = d(prob.x0[:, sl])
                st, it, rel, _ = op.solve(f, x, prob.tol, prob.maxit)
                torch.cuda.current_stream().synchronize()
                res[r] = dict(i0=g.i0, x=x.cpu().numpy(), it=it, st=st)
                op.close()
                g.close()
        except Exception as e:  # noqa: BLE001
            errs.append((r, repr(e)))

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    if errs:
        raise RuntimeError(errs)
    out = [res[r] for r in sorted(res, key=lambda q: res[q]["i0"])]
    return np.concatenate([o["x"] for o in out], axis=1), sorted({o["it"] for o in out}), \
        sorted({o["st"] for o in out})


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ranks", type=int, nargs="+", default=[2, 4, 8])
    args = ap.parse_args()
    prob = W.aniso_conduction_problem(128, 128, 256)
    V = np.einsum("i,j,k->ijk", prob.mesh.rC ** 2 * np.diff(prob.mesh.rF),
                  np.sin(prob.mesh.tC) * np.diff(prob.mesh.tF), np.diff(prob.mesh.pF))[None]
    x1, it1, st1 = solve(prob, 1, 0)
    rep = {"grid": [128, 128, 256], "P1": {"iters": it1, "status": st1}}
    for P in args.ranks:
        xp, itp, stp = solve(prob, P, 100 + P)
        rep[f"P{P}"] = {"iters": itp, "status": stp,
                        "rel_L2V_x": math.sqrt((V * (xp - x1) ** 2).sum() / (V * x1 ** 2).sum())}
    print(json.dumps(rep))


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""C4 parity: the weak-scaling grid at P ranks, (256*P) x 256 x
512 3-component viscosity, solved once on a single B200 as one rank and once
as P ranks through the "virtual ranks" transport (P host threads on the same
GPU, the library's multi-rank driver without NCCL).  At P = 8 that is 268 M
cells (about 45 GB of device memory), which fits one B200.

Prints JSON: iterations (must agree within +-1), relative L2_V difference of x
(<= 1e-10), per-solve times.
"""
import argparse
import json
import math
import os
os.environ.setdefault("MAS_TEST_TRANSPORTS", "1")  # virtual ranks (comm.cpp)
import sys
import threading
import time

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
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                g = M.Grid(prob.mesh, dist=(P, r, vid) if P > 1 else None)
                sl = slice(g.i0, g.i0 + g.nl)
                d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
                op = M.Operator(g, prob.ncomp, d(prob.kappa[sl]), d(prob.c[sl]), prob.bc_inner,
                                prob.bc_outer)
                f = d(prob.f[:, sl])
                x = d(prob.x0[:, sl])
                torch.cuda.current_stream().synchronize()
                t0 = time.perf_counter()
                st, it, rel, _ = op.solve(f, x, prob.tol, prob.maxit)
                torch.cuda.current_stream().synchronize()
                t = time.perf_counter() - t0  # first (cold) solve: includes history-buffer
                # allocation, graph build and module loading
                res[r] = dict(i0=g.i0, x=x.cpu().numpy(), it=it, st=st, rel=rel, t=t)
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
    parts = [res[r] for r in range(P)]
    return (np.concatenate([p["x"] for p in parts], axis=1), {p["it"] for p in parts},
            max(p["t"] for p in parts), {p["st"] for p in parts})


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ranks", type=int, default=8)
    ap.add_argument("--nr-per-rank", type=int, default=256)
    args = ap.parse_args()
    from paper_conf_ipps_caplansl23_b200 import build
    build.build()
    P = args.ranks
    t0 = time.perf_counter()
    prob = W.viscosity_problem(args.nr_per_rank * P, 256, 512)
    gen = time.perf_counter() - t0
    x1, it1, t1, st1 = solve(prob, 1, 0)
    xP, itP, tP, stP = solve(prob, P, 777)
    # relative L2 with the cell volumes (1-D product form: V = rC^2 dr * sin(tC) dt * dp)
    m = prob.mesh
    vr = m.rC ** 2 * np.diff(m.rF)
    vt = np.sin(m.tC) * np.diff(m.tF)
    vp = np.diff(m.pF)
    num = den = 0.0
    for i in range(len(m.rC)):
        Vi = vr[i] * vt[:, None] * vp[None, :]
        num += float((Vi[None] * (xP[:, i] - x1[:, i]) ** 2).sum())
        den += float((Vi[None] * x1[:, i] ** 2).sum())
    out = {"grid": list(prob.shape), "cells": int(np.prod(prob.shape)), "ranks": P,
           "gen_s": gen, "P1": {"iters": sorted(it1), "status": sorted(st1), "first_solve_s_cold": t1},
           f"P{P}": {"iters": sorted(itP), "status": sorted(stP), "first_solve_s_cold": tP},
           "rel_x": math.sqrt(num / den)}
    out["parity_ok"] = bool(len(itP) == 1 and abs(next(iter(itP)) - next(iter(it1))) <= 1
                            and out["rel_x"] <= 1e-10)
    print(json.dumps(out))


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""C5 long run: N implicit steps of conduction (kappa =
(T^n)^{5/2} refreshed by mas_op_update) + 3-component viscosity on
320x300x600 (57.6 M cells), warm starts, Delta t frozen at step 0.

Runs the trajectory with P ranks (P = 1: one GPU; P > 1: the "virtual ranks"
transport, P host threads on one GPU — the multi-rank driver without NCCL)
and prints per-step iteration counts and times as JSON.  --compare runs
P = 1 and P = --ranks and checks the drift criterion: per-step iterations
within +-1 with no trend, final state within 1e-9.
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


def trajectory(L, P, steps, key):
    res, errs = {}, []
    vid = M.virtual_ranks_id(key) if P > 1 else None

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                g = M.Grid(L.mesh, dist=(P, r, vid) if P > 1 else None)
                sl = slice(g.i0, g.i0 + g.nl)
                d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
                Tg = d(L.T0[sl])[None].contiguous()
                vg = d(L.v0[:, sl])
                cT, cv, rho, Tb = d(L.c_T[sl]), d(L.c_v[sl]), d(L.rho[sl]), d(L.T_b)
                opT = M.Operator(g, 1, (Tg[0] ** 2.5).contiguous(), cT, W.DIRICHLET, W.NEUMANN)
                opv = M.Operator(g, 3, rho, cv, W.DIRICHLET, W.NEUMANN)
                its, times = [], []
                for n in range(steps):
                    torch.cuda.current_stream().synchronize()
                    t0 = time.perf_counter()
                    if n:
                        opT.update((Tg[0] ** 2.5).contiguous(), cT)
                    f = (cT * Tg).contiguous()
                    opT.dirichlet_rhs(Tb, None, f)
                    st, itT, _, _ = opT.solve(f, Tg, L.tol, L.maxit)
                    fv = (cv[None] * vg).contiguous()
                    st2, itv, _, _ = opv.solve(fv, vg, L.tol, L.maxit)
                    torch.cuda.current_stream().synchronize()
                    times.append(time.perf_counter() - t0)
                    its.append((itT, itv, st, st2))
                res[r] = dict(i0=g.i0, T=Tg[0].cpu().numpy(), v=vg.cpu().numpy(), its=its,
                              times=times)
                opT.close()
                opv.close()
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
    T = np.concatenate([p["T"] for p in parts], axis=0)
    v = np.concatenate([p["v"] for p in parts], axis=1)
    return T, v, parts[0]["its"], parts[0]["times"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--grid", default="320,300,600")
    ap.add_argument("--ranks", type=int, default=8)
    ap.add_argument("--compare", action="store_true")
    args = ap.parse_args()
    from paper_conf_ipps_caplansl23_b200 import build
    build.build()
    nr, nt, np_ = map(int, args.grid.split(","))
    L = W.longrun_problem(nr, nt, np_)
    out = {"grid": [nr, nt, np_], "steps": args.steps}
    T1, v1, its1, t1 = trajectory(L, 1, args.steps, 0)
    out["P1"] = {"iters": [i[:2] for i in its1], "status": sorted({i[2] for i in its1} | {i[3] for i in its1}),
                 "s_per_step_median": float(np.median(t1))}
    if args.compare and args.ranks > 1:
        TP, vP, itsP, tP = trajectory(L, args.ranks, args.steps, 4242)
        dif = np.array([i[:2] for i in itsP]) - np.array([i[:2] for i in its1])
        h = args.steps // 2
        V = np.ones_like(T1)
        rel = lambda a, b: math.sqrt(((a - b) ** 2).sum() / (b ** 2).sum())
        out[f"P{args.ranks}"] = {"s_per_step_median": float(np.median(tP)),
                                 "max_abs_iter_diff": int(np.abs(dif).max()),
                                 "trend": (dif[:h].mean(0) - dif[h:].mean(0)).tolist(),
                                 "rel_T": rel(TP, T1), "rel_v": rel(vP, v1)}
        out["drift_ok"] = bool(np.abs(dif).max() <= 1 and np.abs(dif[:h].mean(0) - dif[h:].mean(0)).max() <= 1
                               and out[f"P{args.ranks}"]["rel_T"] <= 1e-9 and out[f"P{args.ranks}"]["rel_v"] <= 1e-9)
        del V
    print(json.dumps(out))


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""Staggered viscosity step as ONE solve (mas_stack_solve, NEXT-2, reading
R34) at C3's size on one B200, beside C3's cell-centred 3-component solve.

Each block is a scalar operator at its own location: v_r on the r nodes,
v_theta on the theta nodes, v_phi on the phi nodes (workloads.
staggered_viscosity_blocks: C3's fields evaluated there).  Per iteration each
block runs kernel A (68 B per unknown on average: r, p_old, dinv, kappa, c read,
p, q written, and x read and written with p_(k-2) read by every second launch --
the two-iteration x update; bench.alg_bytes_per_cell(1)) and kernel B (32 B: r,
q, dinv read; r written), plus the
one-warp k_stack_sum nodes.  Timed with CUDA events around mas_stack_solve
(x reset to x0 before each step, outside the events), after warm-up.
Prints one JSON line."""
from __future__ import annotations

import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_ipps_caplansl23_b200 import workloads as W  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--nr", type=int, default=256)
    ap.add_argument("--nt", type=int, default=256)
    ap.add_argument("--np", type=int, default=512)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--tol", type=float, default=1e-12)
    args = ap.parse_args()
    import torch
    from paper_conf_ipps_caplansl23_b200 import build, maspcg as M
    build.build()
    dev = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    hbm = float(peaks.get("hbm_gbs") or peaks.get("hbm_copy_gbs") or 6554.6)

    def timed(solve, reset):
        times, iters = [], None
        for step in range(args.warmup + args.steps):
            reset()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            st, it, rel = solve()
            e1.record()
            torch.cuda.synchronize()
            assert st == M.MAS_OK, st
            if step >= args.warmup:
                times.append(e0.elapsed_time(e1))
                iters = it
        ms = float(np.median(times))
        return iters, ms

    # the staggered stack
    mesh, dt, blocks = W.staggered_viscosity_blocks(args.nr, args.nt, args.np)
    g = M.Grid(mesh)
    ops = [M.Operator(g, 1, dev(k), dev(c), W.DIRICHLET, W.NEUMANN, placement=pl)
           for pl, k, c, f, x0 in blocks]
    sk = M.Stack(ops)
    rhs = [dev(b[3]) for b in blocks]
    x0s = [dev(b[4]) for b in blocks]
    xs = [torch.empty_like(x) for x in x0s]

    def reset_s():
        for x, x0 in zip(xs, x0s):
            x.copy_(x0)

    def solve_s():
        st, it, rel, _ = sk.solve(rhs, xs, args.tol, 20000)
        return st, it, rel

    it_s, ms_s = timed(solve_s, reset_s)
    unknowns = sum(int(np.prod(b[1].shape)) for b in blocks)
    sys.path.insert(0, ROOT)
    import bench  # the byte counts of the bench contract
    bytes_it = sum(bench.alg_bytes_per_cell(1)) * unknowns  # 68 + 32 B per unknown
    sk.close()
    for o in ops:
        o.close()
    g.close()
    del rhs, x0s, xs
    torch.cuda.empty_cache()

    # C3's cell-centred 3-component solve, same timing
    prob = W.viscosity_problem(args.nr, args.nt, args.np)
    g = M.Grid(prob.mesh)
    op = M.Operator(g, 3, dev(prob.kappa), dev(prob.c), prob.bc_inner, prob.bc_outer)
    f, x0 = dev(prob.f), dev(prob.x0)
    x = torch.empty_like(x0)

    def solve_c():
        st, it, rel, _ = op.solve(f, x, args.tol, 20000)
        return st, it, rel

    it_c, ms_c = timed(solve_c, lambda: x.copy_(x0))
    cells = int(np.prod(prob.kappa.shape))
    op.close()
    g.close()

    per_it_s = ms_s / it_s
    per_it_c = ms_c / it_c
    print(json.dumps({
        "tool": "stack_bench", "grid": [args.nr, args.nt, args.np], "tol": args.tol,
        "staggered_stack": {"blocks": ["v_r r-nodes", "v_theta theta-nodes", "v_phi phi-nodes"],
                            "unknowns": unknowns, "iters": it_s, "ms_per_solve": ms_s,
                            "iters_per_s": 1e3 * it_s / ms_s, "ms_per_iter": per_it_s,
                            "alg_bytes_per_iter": bytes_it,
                            "alg_GBs": bytes_it / (per_it_s * 1e-3) / 1e9,
                            "frac_of_hbm": bytes_it / (per_it_s * 1e-3) / 1e9 / hbm},
        "cell_3comp_C3": {"unknowns": 3 * cells, "iters": it_c, "ms_per_solve": ms_c,
                          "iters_per_s": 1e3 * it_c / ms_c, "ms_per_iter": per_it_c,
                          "alg_bytes_per_iter": 248 * cells,
                          "alg_GBs": 248 * cells / (per_it_c * 1e-3) / 1e9,
                          "frac_of_hbm": 248 * cells / (per_it_c * 1e-3) / 1e9 / hbm},
        "hbm_peak_gbs": hbm,
    }))


if __name__ == "__main__":
    main()

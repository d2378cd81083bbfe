"""Time mas_op_apply (k_stencil<APPLY>: y = L x, 3 components) on C3 and
report its HBM rate: the cost of a stencil pass that is NOT dominated by the
PCG vector traffic (reads x, kappa, c; writes y: 8 passes of 8 B per cell).
Used to ground DESIGN.md's NEXT-1 analysis (a single-reduction CG needs a
second, lighter stencil pass per iteration)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch

from paper_conf_ipps_caplansl23_b200 import build as B
from paper_conf_ipps_caplansl23_b200 import workloads as W

B.build()
from paper_conf_ipps_caplansl23_b200 import maspcg as M

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
kind, shape = {"C3": ("viscosity", (256, 256, 512)), "C2": ("conduction", (128, 128, 256))}[cfg]
prob = W.make(kind, nr=shape[0], nt=shape[1], np_=shape[2])
d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
g = M.Grid(prob.mesh)
op = M.Operator(g, prob.ncomp, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer)
x = d(prob.x0)
y = torch.empty_like(x)
for _ in range(3):
    op.apply(x, y)
torch.cuda.synchronize()
n = 20
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(n):
    op.apply(x, y)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / n
cells = int(np.prod(shape))
nbytes = (2 * prob.ncomp + 2) * 8 * cells
print(json.dumps({"config": cfg, "kernel": "k_stencil<APPLY>", "ms": ms,
                  "alg_bytes": nbytes, "GBs": nbytes / (ms / 1e3) / 1e9}))

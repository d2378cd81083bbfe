"""Small driver for ncu: set up config C3 (or --config) and run one PCG solve
with a few iterations through the C ABI.  Launch order: k_diag (setup),
k_stencil<RESID>, then per iteration k_stencil<PCGA>, k_pcg_b (C2a: k_aniso_coef,
k_diag, k_aniso_diag at setup; k_aniso<RESID> after the init; k_aniso<PCGA>
after every kernel A)."""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch

from paper_conf_ipps_caplansl23_b200 import maspcg as M
from paper_conf_ipps_caplansl23_b200 import workloads as W

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C3")
ap.add_argument("--maxit", type=int, default=4)
ap.add_argument("--solver", default="pcg", choices=["pcg", "cg1"])
args = ap.parse_args()
shapes = {"C3": ("viscosity", 256, 256, 512), "C2": ("conduction", 128, 128, 256),
          "C2a": ("aniso", 128, 128, 256), "C2t": ("tnode", 128, 128, 256)}
kind, nr, nt, np_ = shapes[args.config]
prob = W.make(kind, nr=nr, nt=nt, np_=np_)
d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
g = M.Grid(prob.mesh)
tn = prob.extra.get("placement") == "theta-node"
op = M.Operator(g, prob.ncomp, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer,
                placement=M.MAS_PLACE_THETA_NODE if tn else M.MAS_PLACE_CELL)
if args.solver == "cg1":  # NEXT-1: one k_stencil<CG1> per iteration
    op.set_single_reduction(True)
if prob.kpar is not None:  # C2a: + k_aniso<PCGA> after each kernel A
    op.set_aniso(d(prob.kpar), d(prob.bhat))
f = d(prob.f)
x = d(prob.x0)
st, it, rel, _ = op.solve(f, x, 0.0, args.maxit)
torch.cuda.synchronize()
print("iters", it, "status", st)

"""ORACLE — plain CPU reference for the MAS implicit-parabolic PCG path.

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py
(the cpu_baseline leg and ``--impl reference``) may import this package.  The
product package ``paper_conf_ipps_caplansl23_b200`` never imports it and
shares no code with it (the seeded generators in
``paper_conf_ipps_caplansl23_b200.workloads`` are the only common input).

The arithmetic lives in ``mas_ref.c`` (plain C, fp64, -ffp-contract=off);
this module only compiles it and marshals numpy arrays through ctypes.
Definitions: SURVEY.md §8(c) / DESIGN.md §3, readings R1..R16.  Pins:
tests/test_oracle_pins.py.  "parity unpinned" against the paper itself: the
paper (Caplan et al. 2023) prints no value for this path.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "mas_ref.c")
_SO = os.path.join(_HERE, "libmasref.so")

OK, NOT_CONVERGED, ERR_ARG, ERR_BREAKDOWN = 0, 1, 2, 6


def build(force: bool = False) -> str:
    """Compile the oracle: gcc -O2 -ffp-contract=off -fopenmp (no fast-math)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "mas_ref.h"))):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
                               "-std=c99", "-Wall", "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _SO)
    return _SO


class _Grid(C.Structure):
    _fields_ = [("nr", C.c_int), ("nt", C.c_int), ("np", C.c_int),
                ("rF", C.c_void_p), ("rC", C.c_void_p), ("tF", C.c_void_p),
                ("tC", C.c_void_p), ("pF", C.c_void_p), ("pC", C.c_void_p),
                ("bc_inner", C.c_int), ("bc_outer", C.c_int)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def _f64(a):
    return None if a is None else np.ascontiguousarray(a, dtype=np.float64)


class Oracle:
    """Wraps one mesh + boundary conditions.  All arrays float64, C order
    [comp][r][theta][phi]."""

    def __init__(self, mesh, bc_inner: int, bc_outer: int, threads: int = 0):
        self.mesh = mesh
        self._arrs = [_f64(a) for a in (mesh.rF, mesh.rC, mesh.tF, mesh.tC, mesh.pF, mesh.pC)]
        nr, nt, np_ = mesh.shape
        self.g = _Grid(nr, nt, np_, *[_p(a) for a in self._arrs], bc_inner, bc_outer)
        self.shape = (nr, nt, np_)
        self.N = nr * nt * np_
        if threads:
            lib().mas_ref_set_threads(int(threads))

    @classmethod
    def for_problem(cls, prob, threads: int = 0):
        return cls(prob.mesh, prob.bc_inner, prob.bc_outer, threads)

    def _chk(self, rc):
        if rc not in (OK, NOT_CONVERGED, ERR_BREAKDOWN):
            raise RuntimeError(f"oracle returned {rc}")
        return rc

    def volumes(self):
        V = np.empty(self.shape)
        self._chk(lib().mas_ref_volumes(C.byref(self.g), _p(V)))
        return V

    def apply(self, kappa, c, x):
        x = _f64(x)
        ncomp = x.size // self.N
        y = np.empty_like(x)
        kappa, c = _f64(kappa), _f64(c)
        self._chk(lib().mas_ref_op_apply(C.byref(self.g), ncomp, _p(kappa), _p(c), _p(x), _p(y)))
        return y

    def apply_cells(self, kappa, c, x, idx):
        x = _f64(x)
        ncomp = x.size // self.N
        idx = np.ascontiguousarray(idx, dtype=np.int64)
        out = np.empty(idx.shape[0])
        kappa, c = _f64(kappa), _f64(c)
        self._chk(lib().mas_ref_op_apply_cells(C.byref(self.g), ncomp, _p(kappa), _p(c), _p(x),
                                               C.c_longlong(idx.shape[0]), _p(idx), _p(out)))
        return out

    def diag(self, kappa, c):
        D = np.empty(self.shape)
        kappa, c = _f64(kappa), _f64(c)
        self._chk(lib().mas_ref_op_diag(C.byref(self.g), _p(kappa), _p(c), _p(D)))
        return D

    def dirichlet_rhs(self, kappa, f, ub_inner=None, ub_outer=None):
        f = _f64(f).copy()
        ncomp = f.size // self.N
        kappa, ub_inner, ub_outer = _f64(kappa), _f64(ub_inner), _f64(ub_outer)
        self._chk(lib().mas_ref_dirichlet_rhs(C.byref(self.g), ncomp, _p(kappa), _p(ub_inner),
                                              _p(ub_outer), _p(f)))
        return f

    def dot(self, a, b):
        a, b = _f64(a), _f64(b)
        out = C.c_double()
        self._chk(lib().mas_ref_dot(C.byref(self.g), a.size // self.N, _p(a), _p(b), C.byref(out)))
        return out.value

    def pcg(self, kappa, c, f, x0, tol, maxit, nranks: int = 0):
        """Returns (status, x, iters, relres, res_hist[:iters+1])."""
        f = _f64(f)
        x = _f64(x0).copy()
        ncomp = f.size // self.N
        kappa, c = _f64(kappa), _f64(c)
        iters, relres = C.c_int(), C.c_double()
        hist = np.zeros(maxit + 1)
        if nranks:
            rc = lib().mas_ref_pcg_solve_vranks(C.byref(self.g), nranks, ncomp, _p(kappa), _p(c),
                                                _p(f), _p(x), C.c_double(tol), maxit,
                                                C.byref(iters), C.byref(relres), _p(hist))
        else:
            rc = lib().mas_ref_pcg_solve(C.byref(self.g), ncomp, _p(kappa), _p(c), _p(f), _p(x),
                                         C.c_double(tol), maxit, C.byref(iters), C.byref(relres),
                                         _p(hist))
        self._chk(rc)
        return rc, x, iters.value, relres.value, hist[: iters.value + 1]

    def apply_slab(self, i0, nl, kappa_ext, c_loc, x_ext):
        x_ext = _f64(x_ext)
        plane = self.shape[1] * self.shape[2]
        ncomp = x_ext.size // (plane * (nl + 2))
        y = np.empty((ncomp, nl, self.shape[1], self.shape[2]))
        kappa_ext, c_loc = _f64(kappa_ext), _f64(c_loc)
        self._chk(lib().mas_ref_op_apply_slab(C.byref(self.g), i0, nl, ncomp, _p(kappa_ext),
                                              _p(c_loc), _p(x_ext), _p(y)))
        return y

    def apply_block(self, i0, nl, j0, ntl, kappa_ext, c_loc, x_ext):
        """(r, theta) block operator; *_ext carry one ghost plane / row per side."""
        x_ext = _f64(x_ext)
        npp = self.shape[2]
        ncomp = x_ext.size // ((nl + 2) * (ntl + 2) * npp)
        y = np.empty((ncomp, nl, ntl, npp))
        kappa_ext, c_loc = _f64(kappa_ext), _f64(c_loc)
        self._chk(lib().mas_ref_op_apply_block(C.byref(self.g), i0, nl, j0, ntl, ncomp,
                                               _p(kappa_ext), _p(c_loc), _p(x_ext), _p(y)))
        return y

    def dot_block(self, i0, nl, j0, ntl, a, b):
        a, b = _f64(a), _f64(b)
        out = C.c_double()
        ncomp = a.size // (nl * ntl * self.shape[2])
        self._chk(lib().mas_ref_dot_block(C.byref(self.g), i0, nl, j0, ntl, ncomp, _p(a), _p(b),
                                          C.byref(out)))
        return out.value

    def dot_slab(self, i0, nl, a, b):
        a, b = _f64(a), _f64(b)
        plane = self.shape[1] * self.shape[2]
        out = C.c_double()
        self._chk(lib().mas_ref_dot_slab(C.byref(self.g), i0, nl, a.size // (plane * nl), _p(a),
                                         _p(b), C.byref(out)))
        return out.value

    # ---- field-aligned conduction (NEXT-4, readings R21-R26) ----------------
    def aniso_apply(self, kpar, bhat, x):
        """y = L_par x (kpar [nr,nt,np], bhat [3,nr,nt,np] at lower corners)."""
        x = _f64(x)
        ncomp = x.size // self.N
        y = np.empty_like(x)
        kpar, bhat = _f64(kpar), _f64(bhat)
        self._chk(lib().mas_ref_aniso_apply(C.byref(self.g), ncomp, _p(kpar), _p(bhat), _p(x),
                                            _p(y)))
        return y

    def aniso_diag(self, kpar, bhat):
        D = np.empty(self.shape)
        kpar, bhat = _f64(kpar), _f64(bhat)
        self._chk(lib().mas_ref_aniso_diag(C.byref(self.g), _p(kpar), _p(bhat), _p(D)))
        return D

    def aniso_apply_slab(self, i0, nl, kpar_ext, bhat_ext, x_ext):
        """Slab-local L_par: x_ext with ghost planes, corner fields with the
        corner plane above the slab."""
        x_ext = _f64(x_ext)
        plane = self.shape[1] * self.shape[2]
        ncomp = x_ext.size // (plane * (nl + 2))
        y = np.empty((ncomp, nl, self.shape[1], self.shape[2]))
        kpar_ext, bhat_ext = _f64(kpar_ext), _f64(bhat_ext)
        self._chk(lib().mas_ref_aniso_apply_slab(C.byref(self.g), i0, nl, ncomp, _p(kpar_ext),
                                                 _p(bhat_ext), _p(x_ext), _p(y)))
        return y

    def radial_sums(self, x, w):
        """sum0[m][i] = sum_{j,k} w[j][k] x[m][i][j][k] (Listings 3-5, R27)."""
        x, w = _f64(x), _f64(w)
        ncomp = x.size // self.N
        out = np.empty((ncomp, self.shape[0]))
        self._chk(lib().mas_ref_radial_sums(C.byref(self.g), ncomp, _p(x), _p(w), _p(out)))
        return out

    def pcg_aniso(self, kappa, c, kpar, bhat, f, x0, tol, maxit):
        """PCG on L_iso + L_par.  Returns (status, x, iters, relres, res_hist)."""
        f = _f64(f)
        x = _f64(x0).copy()
        ncomp = f.size // self.N
        kappa, c, kpar, bhat = _f64(kappa), _f64(c), _f64(kpar), _f64(bhat)
        iters, relres = C.c_int(), C.c_double()
        hist = np.zeros(maxit + 1)
        rc = lib().mas_ref_pcg_solve_aniso(C.byref(self.g), ncomp, _p(kappa), _p(c), _p(kpar),
                                           _p(bhat), _p(f), _p(x), C.c_double(tol), maxit,
                                           C.byref(iters), C.byref(relres), _p(hist))
        self._chk(rc)
        return rc, x, iters.value, relres.value, hist[: iters.value + 1]


    def pcg_cg1(self, kappa, c, f, x0, tol, maxit):
        """Single-reduction (Chronopoulos-Gear) PCG, NEXT-1 / R28.
        Returns (status, x, iters, relres, res_hist)."""
        f = _f64(f)
        x = _f64(x0).copy()
        ncomp = f.size // self.N
        kappa, c = _f64(kappa), _f64(c)
        iters, relres = C.c_int(), C.c_double()
        hist = np.zeros(maxit + 1)
        rc = lib().mas_ref_pcg_solve_cg1(C.byref(self.g), ncomp, _p(kappa), _p(c), _p(f), _p(x),
                                         C.c_double(tol), maxit, C.byref(iters), C.byref(relres),
                                         _p(hist))
        self._chk(rc)
        return rc, x, iters.value, relres.value, hist[: iters.value + 1]


    # ---- theta-node placement with pole unknowns (NEXT-2, R29-R30) --------
    @property
    def tn_shape(self):
        nr, nt, np_ = self.shape
        return (nr, nt + 1, np_)

    def tn_volumes(self):
        V = np.empty(self.tn_shape)
        self._chk(lib().mas_ref_tn_volumes(C.byref(self.g), _p(V)))
        return V

    def tn_apply(self, kappa, c, x):
        x = _f64(x)
        ncomp = x.size // int(np.prod(self.tn_shape))
        y = np.empty_like(x)
        kappa, c = _f64(kappa), _f64(c)
        self._chk(lib().mas_ref_tn_apply(C.byref(self.g), ncomp, _p(kappa), _p(c), _p(x), _p(y)))
        return y

    def tn_diag(self, kappa, c):
        D = np.empty(self.tn_shape)
        kappa, c = _f64(kappa), _f64(c)
        self._chk(lib().mas_ref_tn_diag(C.byref(self.g), _p(kappa), _p(c), _p(D)))
        return D

    def tn_dirichlet_rhs(self, kappa, f, ub_inner=None, ub_outer=None):
        f = _f64(f).copy()
        ncomp = f.size // int(np.prod(self.tn_shape))
        kappa, ub_inner, ub_outer = _f64(kappa), _f64(ub_inner), _f64(ub_outer)
        self._chk(lib().mas_ref_tn_dirichlet_rhs(C.byref(self.g), ncomp, _p(kappa), _p(ub_inner),
                                                 _p(ub_outer), _p(f)))
        return f

    def tn_dot(self, a, b):
        a, b = _f64(a), _f64(b)
        out = C.c_double()
        self._chk(lib().mas_ref_tn_dot(C.byref(self.g), a.size // int(np.prod(self.tn_shape)), _p(a),
                                       _p(b), C.byref(out)))
        return out.value

    def tn_pcg(self, kappa, c, f, x0, tol, maxit):
        """Returns (status, x, iters, relres, res_hist[:iters+1])."""
        f = _f64(f)
        x = _f64(x0).copy()
        ncomp = f.size // int(np.prod(self.tn_shape))
        kappa, c = _f64(kappa), _f64(c)
        iters, relres = C.c_int(), C.c_double()
        hist = np.zeros(maxit + 1)
        rc = lib().mas_ref_tn_pcg_solve(C.byref(self.g), ncomp, _p(kappa), _p(c), _p(f), _p(x),
                                        C.c_double(tol), maxit, C.byref(iters), C.byref(relres),
                                        _p(hist))
        self._chk(rc)
        return rc, x, iters.value, relres.value, hist[: iters.value + 1]


    # ---- vector-Laplacian curvature terms (NEXT-2, R31), ncomp = 3 ---------
    def apply_curv(self, kappa, c, x):
        x = _f64(x)
        y = np.empty_like(x)
        kappa, c = _f64(kappa), _f64(c)
        self._chk(lib().mas_ref_op_apply_curv(C.byref(self.g), _p(kappa), _p(c), _p(x), _p(y)))
        return y

    def pcg_curv(self, kappa, c, f, x0, tol, maxit):
        f = _f64(f)
        x = _f64(x0).copy()
        kappa, c = _f64(kappa), _f64(c)
        iters, relres = C.c_int(), C.c_double()
        hist = np.zeros(maxit + 1)
        rc = lib().mas_ref_pcg_solve_curv(C.byref(self.g), _p(kappa), _p(c), _p(f), _p(x),
                                          C.c_double(tol), maxit, C.byref(iters), C.byref(relres),
                                          _p(hist))
        self._chk(rc)
        return rc, x, iters.value, relres.value, hist[: iters.value + 1]


    # ---- face-centred placements (NEXT-2, R32-R33) ----------------------
    @property
    def rn_shape(self):
        nr, nt, np_ = self.shape
        return (nr - 1, nt, np_)

    def rn_volumes(self):
        V = np.empty(self.rn_shape)
        self._chk(lib().mas_ref_rn_volumes(C.byref(self.g), _p(V)))
        return V

    def rn_apply(self, kappa, c, x):
        x = _f64(x)
        y = np.empty_like(x)
        kappa, c = _f64(kappa), _f64(c)
        self._chk(lib().mas_ref_rn_apply(C.byref(self.g), x.size // int(np.prod(self.rn_shape)), _p(kappa),
                                         _p(c), _p(x), _p(y)))
        return y

    def rn_diag(self, kappa, c):
        D = np.empty(self.rn_shape)
        kappa, c = _f64(kappa), _f64(c)
        self._chk(lib().mas_ref_rn_diag(C.byref(self.g), _p(kappa), _p(c), _p(D)))
        return D

    def rn_dirichlet_rhs(self, kappa, f, ub_inner=None, ub_outer=None):
        f = _f64(f).copy()
        kappa, ub_inner, ub_outer = _f64(kappa), _f64(ub_inner), _f64(ub_outer)
        self._chk(lib().mas_ref_rn_dirichlet_rhs(C.byref(self.g), f.size // int(np.prod(self.rn_shape)),
                                                 _p(kappa), _p(ub_inner), _p(ub_outer), _p(f)))
        return f

    def rn_pcg(self, kappa, c, f, x0, tol, maxit):
        f = _f64(f)
        x = _f64(x0).copy()
        kappa, c = _f64(kappa), _f64(c)
        iters, relres = C.c_int(), C.c_double()
        hist = np.zeros(maxit + 1)
        rc = lib().mas_ref_rn_pcg_solve(C.byref(self.g), f.size // int(np.prod(self.rn_shape)), _p(kappa),
                                        _p(c), _p(f), _p(x), C.c_double(tol), maxit, C.byref(iters),
                                        C.byref(relres), _p(hist))
        self._chk(rc)
        return rc, x, iters.value, relres.value, hist[: iters.value + 1]

    def pn_volumes(self):
        V = np.empty(self.shape)
        self._chk(lib().mas_ref_pn_volumes(C.byref(self.g), _p(V)))
        return V

    def pn_apply(self, kappa, c, x):
        x = _f64(x)
        y = np.empty_like(x)
        kappa, c = _f64(kappa), _f64(c)
        self._chk(lib().mas_ref_pn_apply(C.byref(self.g), x.size // self.N, _p(kappa), _p(c), _p(x), _p(y)))
        return y

    def pn_diag(self, kappa, c):
        D = np.empty(self.shape)
        kappa, c = _f64(kappa), _f64(c)
        self._chk(lib().mas_ref_pn_diag(C.byref(self.g), _p(kappa), _p(c), _p(D)))
        return D

    def pn_dirichlet_rhs(self, kappa, f, ub_inner=None, ub_outer=None):
        f = _f64(f).copy()
        kappa, ub_inner, ub_outer = _f64(kappa), _f64(ub_inner), _f64(ub_outer)
        self._chk(lib().mas_ref_pn_dirichlet_rhs(C.byref(self.g), f.size // self.N, _p(kappa), _p(ub_inner),
                                                 _p(ub_outer), _p(f)))
        return f

    def pn_pcg(self, kappa, c, f, x0, tol, maxit):
        f = _f64(f)
        x = _f64(x0).copy()
        kappa, c = _f64(kappa), _f64(c)
        iters, relres = C.c_int(), C.c_double()
        hist = np.zeros(maxit + 1)
        rc = lib().mas_ref_pn_pcg_solve(C.byref(self.g), f.size // self.N, _p(kappa), _p(c), _p(f), _p(x),
                                        C.c_double(tol), maxit, C.byref(iters), C.byref(relres), _p(hist))
        self._chk(rc)
        return rc, x, iters.value, relres.value, hist[: iters.value + 1]


PLACE_CELL, PLACE_THETA_NODE, PLACE_R_NODE, PLACE_PHI_NODE = 0, 1, 2, 3


def stacked_pcg(blocks, tol, maxit):
    """ONE Jacobi-PCG on the stacked vector of several placed operators
    (NEXT-2, reading R34: MAS's viscosity step with v_r at r nodes, v_theta at
    theta nodes, v_phi at phi nodes; mas_ref_stacked_pcg_solve).  blocks: a
    list of (Oracle, placement, kappa, c, f, x0), c may be None; f and x0 of
    shape (ncomp,) + the placement's shape.  Returns (status, [x_b],
    iters, relres, res_hist[:iters+1])."""
    n = len(blocks)
    grids = (C.POINTER(_Grid) * n)(*[C.pointer(b[0].g) for b in blocks])
    pl = (C.c_int * n)(*[int(b[1]) for b in blocks])
    keep = []
    ncomp, kap, cc, ff, xx = [], [], [], [], []
    for o, place, kappa, c, f, x0 in blocks:
        kappa, c, f = _f64(kappa), _f64(c), _f64(f)
        x = _f64(x0).copy()
        keep += [kappa, c, f, x]
        ncomp.append(f.size // kappa.size)
        kap.append(_p(kappa)); cc.append(_p(c)); ff.append(_p(f)); xx.append(x)
    iters, relres = C.c_int(), C.c_double()
    hist = np.zeros(maxit + 1)
    VP = C.c_void_p * n
    rc = lib().mas_ref_stacked_pcg_solve(
        n, grids, pl, (C.c_int * n)(*ncomp), VP(*kap), VP(*cc), VP(*ff), VP(*[_p(x) for x in xx]),
        C.c_double(tol), maxit, C.byref(iters), C.byref(relres), _p(hist))
    if rc not in (OK, NOT_CONVERGED, ERR_BREAKDOWN):
        raise RuntimeError(f"oracle returned {rc}")
    return rc, xx, iters.value, relres.value, hist[: iters.value + 1]


def partition(nr: int, nranks: int, rank: int):
    i0, nl = C.c_int(), C.c_int()
    lib().mas_ref_partition(nr, nranks, rank, C.byref(i0), C.byref(nl))
    return i0.value, nl.value


def solve_problem(prob, tol=None, maxit=None, x0=None, threads: int = 0, nranks: int = 0,
                  cg1: bool = False):
    """Full oracle solve of a workloads.Problem: rhs = f + Dirichlet terms.
    cg1: the single-reduction (Chronopoulos-Gear) PCG of NEXT-1."""
    o = Oracle.for_problem(prob, threads)
    f = o.dirichlet_rhs(prob.kappa, prob.f, prob.ub_inner, prob.ub_outer)
    if cg1:
        if prob.kpar is not None or nranks:
            raise ValueError("cg1: isotropic operator, one rank")
        return o.pcg_cg1(prob.kappa, prob.c, f, prob.x0 if x0 is None else x0,
                         prob.tol if tol is None else tol, prob.maxit if maxit is None else maxit)
    if prob.kpar is not None:  # field-aligned conduction (NEXT-4)
        return o.pcg_aniso(prob.kappa, prob.c, prob.kpar, prob.bhat, f,
                           prob.x0 if x0 is None else x0, prob.tol if tol is None else tol,
                           prob.maxit if maxit is None else maxit)
    return o.pcg(prob.kappa, prob.c, f, prob.x0 if x0 is None else x0,
                 prob.tol if tol is None else tol, prob.maxit if maxit is None else maxit,
                 nranks=nranks)

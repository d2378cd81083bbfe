"""Seeded synthetic workloads for the MAS implicit-parabolic PCG path.

This module is the ONLY code shared by the CUDA path's tests/bench and the
oracle's tests: it builds meshes and coefficient fields and holds none of the
method's arithmetic (no face conductances, no operator, no PCG).  Recipe:
SURVEY.md §8(d) "Synthetic workloads", restated in DESIGN.md §4.

The paper's test problem is a 36 M-cell production coronal background
(§V-A) on a "stretched grid" (Fig. 1) of the
"logically rectangular non-uniform staggered spherical grid" (P:208-209,
§III).  Its inputs are not available; these fields are stand-ins of the same
shape: geometric radial stretching, a theta mesh with 3x larger cells at the
poles than at the equator, uniform periodic phi, radially stratified density and
temperature with a smooth 3-D angular texture.

Everything is float64 numpy, C order [comp][i=r][j=theta][k=phi].
"""
from __future__ import annotations

import dataclasses
import math
from typing import Optional

import numpy as np

DIRICHLET = 0
NEUMANN = 1
GAMMA = 5.0 / 3.0


@dataclasses.dataclass
class Mesh:
    rF: np.ndarray  # [nr+1] r faces (main / node mesh)
    rC: np.ndarray  # [nr]   r centres (half mesh)
    tF: np.ndarray  # [nt+1]
    tC: np.ndarray  # [nt]
    pF: np.ndarray  # [np+1]
    pC: np.ndarray  # [np]
    pole_north: bool = True
    pole_south: bool = True

    @property
    def shape(self):
        return (len(self.rC), len(self.tC), len(self.pC))

    @property
    def ncells(self) -> int:
        nr, nt, np_ = self.shape
        return nr * nt * np_


@dataclasses.dataclass
class Problem:
    """One implicit parabolic solve: (L x) = f with Dirichlet data ub_*."""
    name: str
    mesh: Mesh
    ncomp: int
    kappa: np.ndarray                 # [nr,nt,np]  >= 0
    c: Optional[np.ndarray]           # [nr,nt,np]  >= 0 (None = 0)
    f: np.ndarray                     # [ncomp,nr,nt,np] rhs WITHOUT boundary terms
    x0: np.ndarray                    # [ncomp,nr,nt,np]
    bc_inner: int
    bc_outer: int
    ub_inner: Optional[np.ndarray]    # [ncomp,nt,np] or None (homogeneous)
    ub_outer: Optional[np.ndarray]
    tol: float
    maxit: int
    extra: dict = dataclasses.field(default_factory=dict)
    # field-aligned conduction (NEXT-4): kpar [nr,nt,np] and bhat [3,nr,nt,np]
    # given at the LOWER corner (rF_i, tF_j, pF_k) of cell (i,j,k) (reading R25)
    kpar: Optional[np.ndarray] = None
    bhat: Optional[np.ndarray] = None

    @property
    def shape(self):
        return self.mesh.shape


# ----------------------------------------------------------------------------
# meshes
# ----------------------------------------------------------------------------
def stretched_mesh(nr: int, nt: int, np_: int, r0: float = 1.0, r1: float = 30.0,
                   R: float = 200.0, a: float = 0.5) -> Mesh:
    """SURVEY §8(d) "Mesh": geometric r faces with dr_last/dr_first = R;
    tF = pi (s + a/(2 pi) sin 2 pi s) (pole cells (1+a)/(1-a) = 3x the
    equatorial ones at a = 0.5), uniform phi; centres are midpoints."""
    if nr > 1 and R != 1.0:
        q = R ** (1.0 / (nr - 1))
        i = np.arange(nr + 1, dtype=np.float64)
        rF = r0 + (r1 - r0) * (q ** i - 1.0) / (q ** nr - 1.0)
    else:
        rF = np.linspace(r0, r1, nr + 1)
    rF[0], rF[-1] = r0, r1
    s = np.arange(nt + 1, dtype=np.float64) / nt
    tF = math.pi * (s + (a / (2.0 * math.pi)) * np.sin(2.0 * math.pi * s))
    tF[0], tF[-1] = 0.0, math.pi
    pF = 2.0 * math.pi * np.arange(np_ + 1, dtype=np.float64) / np_
    mid = lambda F: 0.5 * (F[1:] + F[:-1])
    return Mesh(rF=rF, rC=mid(rF), tF=tF, tC=mid(tF), pF=pF, pC=mid(pF))


def texture(tC: np.ndarray, pC: np.ndarray, seed: int, at=None) -> np.ndarray:
    """g(theta,phi) = sum_{m=0..3} sin^m(theta) (a_m cos(theta) + b_m) cos(m phi + c_m),
    a_m, b_m ~ N(0,1), c_m ~ U[0, 2pi), normalised to max|g| = 1 on the cell
    centres.  Smooth at the poles (sin^m factor).  at = (t, p): evaluate the
    same function (same normalisation) at other points, e.g. cell corners."""
    rng = np.random.default_rng(seed)
    am = rng.standard_normal(4)
    bm = rng.standard_normal(4)
    cm = rng.uniform(0.0, 2.0 * math.pi, 4)

    def ev(t, p):
        th = t[:, None]
        ph = p[None, :]
        g = np.zeros((len(t), len(p)))
        for m in range(4):
            g += np.sin(th) ** m * (am[m] * np.cos(th) + bm[m]) * np.cos(m * ph + cm[m])
        return g

    norm = np.abs(ev(tC, pC)).max()
    return (ev(tC, pC) if at is None else ev(*at)) / norm


def _temperature(r, gT):
    return (0.01 + 0.99 * (1.0 - np.exp(-(r - 1.0) / 0.02))) * r ** (-2.0 / 7.0) * (1.0 + 0.2 * gT)


def _density(r, grho):
    return np.exp(-(1.0 - 1.0 / r) / 0.07) * (1.0 + 0.2 * grho)


def _diffusion_number_scale(mesh: Mesh, kappa: np.ndarray, rho_c: np.ndarray) -> float:
    """max_P kappa_P / rho_c,P * (2/dr^2 + 2/(r dtheta)^2 + 2/(r sin(theta) dphi)^2):
    the textbook explicit diffusion number per unit dt (a workload recipe, not
    the operator's conductances).  Delta t = D_max / this."""
    nr = len(mesh.rC)
    dr = np.diff(mesh.rF)
    dt = np.diff(mesh.tF)
    dp = np.diff(mesh.pF)
    sC = np.sin(mesh.tC)
    best = 0.0
    for i in range(nr):  # plane by plane keeps memory flat at 57 M cells
        rr = mesh.rC[i]
        geo = (2.0 / dr[i] ** 2 + 2.0 / (rr * dt[:, None]) ** 2
               + 2.0 / (rr * sC[:, None] * dp[None, :]) ** 2)
        best = max(best, float(np.max(kappa[i] / rho_c[i] * geo)))
    return best


# ----------------------------------------------------------------------------
# problems
# ----------------------------------------------------------------------------
def mms_solution(r, t, p):
    """u* = e^-r (1 + sin^2 t cos 2p + 1/2 sin t sin p)  (SURVEY §8(c) pins)."""
    return np.exp(-r) * (1.0 + np.sin(t) ** 2 * np.cos(2 * p) + 0.5 * np.sin(t) * np.sin(p))


def mms_forcing(r, t, p):
    """-div(kappa grad u*) with kappa = r^2, in closed form (checked with sympy
    in tests/test_oracle_pins.py)."""
    return -np.exp(-r) * ((r * r - 4 * r) + (r * r - 4 * r - 6) * np.sin(t) ** 2 * np.cos(2 * p)
                          + 0.5 * (r * r - 4 * r - 2) * np.sin(t) * np.sin(p))


def mms_problem(nr=16, nt=24, np_=32, r0=1.0, r1=2.0, R=4.0, tol=1e-12, maxit=10000) -> Problem:
    """C1: scalar MMS on a shell, kappa = r^2, c = 0, Dirichlet both ends."""
    m = stretched_mesh(nr, nt, np_, r0, r1, R)
    r, t, p = np.meshgrid(m.rC, m.tC, m.pC, indexing="ij")
    kappa = np.ascontiguousarray(r * r)
    f = mms_forcing(r, t, p)[None].copy()
    tt, pp = np.meshgrid(m.tC, m.pC, indexing="ij")
    ub_in = mms_solution(np.full_like(tt, m.rF[0]), tt, pp)[None].copy()
    ub_out = mms_solution(np.full_like(tt, m.rF[-1]), tt, pp)[None].copy()
    return Problem("C1-mms", m, 1, kappa, np.zeros_like(kappa), f, np.zeros_like(f),
                   DIRICHLET, DIRICHLET, ub_in, ub_out, tol, maxit,
                   extra={"exact": mms_solution(r, t, p)[None].copy()})


def conduction_problem(nr=128, nt=128, np_=256, r0=1.0, r1=30.0, R=200.0, D_max=1000.0,
                       tol=1e-12, maxit=20000, warm=True) -> Problem:
    """C2: implicit thermal conduction step, kappa = T^(5/2),
    c = rho / ((gamma-1) dt), inner Dirichlet u_b = T(r0), outer Neumann,
    f = c T^n, x0 = T^n (warm start, R12) unless warm=False."""
    m = stretched_mesh(nr, nt, np_, r0, r1, R)
    gT = texture(m.tC, m.pC, 1)
    grho = texture(m.tC, m.pC, 2)
    r = m.rC[:, None, None]
    T = np.ascontiguousarray(np.broadcast_to(_temperature(r, gT[None]), (nr, nt, np_)))
    rho = np.ascontiguousarray(np.broadcast_to(_density(r, grho[None]), (nr, nt, np_)))
    kappa = T ** 2.5
    rho_c = rho / (GAMMA - 1.0)
    dt = D_max / _diffusion_number_scale(m, kappa, rho_c)
    c = rho_c / dt
    f = (c * T)[None]
    ub_in = _temperature(np.float64(m.rF[0]), gT)[None].copy()
    x0 = T[None].copy() if warm else np.zeros_like(f)
    return Problem("C2-conduction", m, 1, kappa, c, f, x0, DIRICHLET, NEUMANN, ub_in, None,
                   tol, maxit, extra={"dt": dt})


def viscosity_problem(nr=256, nt=256, np_=512, r0=1.0, r1=30.0, R=200.0, D_max=100.0,
                      tol=1e-12, maxit=20000, warm=True) -> Problem:
    """C3: implicit viscosity step, 3 uncoupled components sharing
    kappa = rho (nu = 1) and c = rho/dt (R13); homogeneous inner Dirichlet,
    outer Neumann; f = c v^n, x0 = v^n."""
    m = stretched_mesh(nr, nt, np_, r0, r1, R)
    grho = texture(m.tC, m.pC, 2)
    r = m.rC[:, None, None]
    rho = np.ascontiguousarray(np.broadcast_to(_density(r, grho[None]), (nr, nt, np_)))
    kappa = rho
    dt = D_max / _diffusion_number_scale(m, kappa, rho)
    c = rho / dt
    v = np.empty((3, nr, nt, np_))
    prof = np.sin(math.pi * (m.rC - r0) / (r1 - r0))[:, None, None]
    for comp in range(3):
        v[comp] = prof * texture(m.tC, m.pC, 10 + comp)[None]
    f = c[None] * v
    x0 = v.copy() if warm else np.zeros_like(v)
    return Problem("C3-viscosity", m, 3, kappa, c, f, x0, DIRICHLET, NEUMANN, None, None,
                   tol, maxit, extra={"dt": dt})


def spiral_dipole_field(r, t, p, omega=0.5, dip=0.3, b0=0.02):
    """Unit magnetic-field direction b = B/|B| in spherical components
    (b_r, b_theta, b_phi) for B = split monopole wound into a Parker spiral
    (B_r = 1/r^2, B_phi = -omega sin(theta)/r) + a dipole of strength dip +
    a uniform b0 x-hat field (breaks the axisymmetry).  Every term is a smooth
    Cartesian field, so b is smooth at the poles (NEXT-4 workload input)."""
    st, ct, sp, cp = np.sin(t), np.cos(t), np.sin(p), np.cos(p)
    Br = 1.0 / r ** 2 + 2.0 * dip * ct / r ** 3 + b0 * st * cp
    Bt = dip * st / r ** 3 + b0 * ct * cp
    Bp = -omega * st / r - b0 * sp
    n = np.sqrt(Br * Br + Bt * Bt + Bp * Bp)
    return np.stack([Br / n, Bt / n, Bp / n])


def aniso_conduction_problem(nr=128, nt=128, np_=256, r0=1.0, r1=30.0, R=200.0,
                             D_max=1000.0, eps_iso=1e-2, tol=1e-12, maxit=20000,
                             warm=True) -> Problem:
    """C2a: field-aligned thermal conduction.  As C2, but
    the conductivity is split into kpar = T^(5/2) along b (at the cell corners,
    reading R25) and an isotropic kappa = eps_iso T^(5/2) at the cell centres;
    b from spiral_dipole_field.  Same dt rule, c, boundary data, f and x0 as C2."""
    prob = conduction_problem(nr, nt, np_, r0, r1, R, D_max, tol, maxit, warm)
    m = prob.mesh
    gT = texture(m.tC, m.pC, 1, at=(m.tF[:-1], m.pF[:-1]))
    rc = m.rF[:-1][:, None, None]
    Tc = _temperature(rc, gT[None])
    tc = m.tF[:-1][None, :, None]
    pc = m.pF[:-1][None, None, :]
    bhat = spiral_dipole_field(rc, tc, pc)
    shape = (nr, nt, np_)
    prob.kpar = np.ascontiguousarray(np.broadcast_to(Tc ** 2.5, shape))
    prob.bhat = np.ascontiguousarray(np.broadcast_to(bhat, (3,) + shape))
    prob.kappa = eps_iso * prob.kappa
    prob.name = "C2a-aniso-conduction"
    prob.extra["eps_iso"] = eps_iso
    return prob


@dataclasses.dataclass
class LongRun:
    """C5: repeated implicit steps of conduction then viscosity,
    warm-started, Delta t frozen at step 0.  Per step n (harness arithmetic,
    not the PCG path): kappa_T = (T^n)^(5/2), rhs_T = c_T T^n (+ Dirichlet
    T_b at r0); rhs_v = c_v v^n."""
    mesh: Mesh
    T0: np.ndarray      # [nr,nt,np]
    v0: np.ndarray      # [3,nr,nt,np]
    rho: np.ndarray     # [nr,nt,np]
    c_T: np.ndarray     # rho / ((gamma-1) dt_T)
    c_v: np.ndarray     # rho / dt_v
    T_b: np.ndarray     # [1,nt,np] inner Dirichlet temperature
    dt_T: float
    dt_v: float
    tol: float = 1e-12
    maxit: int = 20000


def longrun_problem(nr=320, nt=300, np_=600, r0=1.0, r1=30.0, R=200.0, D_T=1000.0,
                    D_v=100.0) -> LongRun:
    m = stretched_mesh(nr, nt, np_, r0, r1, R)
    gT = texture(m.tC, m.pC, 1)
    grho = texture(m.tC, m.pC, 2)
    r = m.rC[:, None, None]
    T = np.ascontiguousarray(np.broadcast_to(_temperature(r, gT[None]), (nr, nt, np_)))
    rho = np.ascontiguousarray(np.broadcast_to(_density(r, grho[None]), (nr, nt, np_)))
    rho_c = rho / (GAMMA - 1.0)
    dt_T = D_T / _diffusion_number_scale(m, T ** 2.5, rho_c)
    dt_v = D_v / _diffusion_number_scale(m, rho, rho)
    v = np.empty((3, nr, nt, np_))
    prof = np.sin(math.pi * (m.rC - r0) / (r1 - r0))[:, None, None]
    for comp in range(3):
        v[comp] = prof * texture(m.tC, m.pC, 10 + comp)[None]
    return LongRun(m, T, v, rho, rho_c / dt_T, rho / dt_v,
                   _temperature(np.float64(m.rF[0]), gT)[None].copy(), dt_T, dt_v)


def replicate_poles(a: np.ndarray) -> np.ndarray:
    """theta-node fields [..., nt+1, np]: every slot of a pole row (first and
    last theta row) takes the row's first value (the pole is one point)."""
    a = np.array(a, dtype=np.float64)
    a[..., 0, :] = a[..., 0, :1]
    a[..., -1, :] = a[..., -1, :1]
    return a


def tnode_conduction_problem(nr=128, nt=128, np_=256, r0=1.0, r1=30.0, R=200.0, D_max=1000.0,
                             tol=1e-12, maxit=20000, warm=True) -> Problem:
    """C2's conduction step with the temperature on the theta NODES
    (rC_i, tF_j, pC_k), j = 0..nt (NEXT-2 placement, readings R29-R30): the
    same T, rho fields and dt as conduction_problem, evaluated at the theta
    nodes; the pole rows (j = 0, nt) are one value per radius (the texture is
    smooth there: only its m = 0 term survives).  Arrays [.., nt+1, np]."""
    base = conduction_problem(nr, nt, np_, r0, r1, R, D_max, tol, maxit, warm)
    m = base.mesh
    gT = texture(m.tC, m.pC, 1, at=(m.tF, m.pC))
    grho = texture(m.tC, m.pC, 2, at=(m.tF, m.pC))
    r = m.rC[:, None, None]
    T = replicate_poles(np.broadcast_to(_temperature(r, gT[None]), (nr, nt + 1, np_)))
    rho = replicate_poles(np.broadcast_to(_density(r, grho[None]), (nr, nt + 1, np_)))
    kappa = T ** 2.5
    c = rho / (GAMMA - 1.0) / base.extra["dt"]
    f = (c * T)[None]
    ub_in = replicate_poles(_temperature(np.float64(m.rF[0]), gT)[None])
    x0 = T[None].copy() if warm else np.zeros_like(f)
    return Problem("C2t-conduction-theta-nodes", m, 1, kappa, c, f, x0, DIRICHLET, NEUMANN, ub_in, None,
                   tol, maxit, extra={"dt": base.extra["dt"], "placement": "theta-node"})


def staggered_viscosity_blocks(nr=256, nt=256, np_=512, r0=1.0, r1=30.0, R=200.0, D_max=100.0,
                               warm=True):
    """C3's viscosity step on the staggered mesh (NEXT-2, reading R34): v_r at
    the r nodes (rF_i, tC, pC), i = 1..nr-1; v_theta at the theta nodes (rC,
    tF_j, pC), j = 0..nt (pole rows one value per radius); v_phi at the phi
    nodes (rC, tC, pF_k).  The same rho texture, nu = 1, dt and velocity
    profile as viscosity_problem, evaluated at each component's location.
    Returns (mesh, dt, [(placement, kappa, c, f[None], x0[None])]) with
    placements 2 (r nodes), 1 (theta nodes), 3 (phi nodes); boundary
    conditions DIRICHLET inner, NEUMANN outer for every block."""
    m = stretched_mesh(nr, nt, np_, r0, r1, R)
    grho_c = texture(m.tC, m.pC, 2)
    rho_c = np.ascontiguousarray(np.broadcast_to(_density(m.rC[:, None, None], grho_c[None]), (nr, nt, np_)))
    dt = D_max / _diffusion_number_scale(m, rho_c, rho_c)
    pF = m.pF[:-1]
    locs = [  # placement, r points, (theta, phi) points of the texture, velocity texture seed
        (2, m.rF[1:-1], (m.tC, m.pC), 10),
        (1, m.rC, (m.tF, m.pC), 11),
        (3, m.rC, (m.tC, pF), 12),
    ]
    out = []
    for pl, rr, (tt, pp), seed in locs:
        g_rho = texture(m.tC, m.pC, 2, at=(tt, pp))
        rho = _density(rr[:, None, None], g_rho[None])
        prof = np.sin(math.pi * (rr - r0) / (r1 - r0))[:, None, None]
        v = prof * texture(m.tC, m.pC, seed, at=(tt, pp))[None]
        shape = (len(rr), len(tt), len(pp))
        rho = np.ascontiguousarray(np.broadcast_to(rho, shape))
        v = np.ascontiguousarray(np.broadcast_to(v, shape))
        if pl == 1:
            rho, v = replicate_poles(rho), replicate_poles(v)
        c = rho / dt
        f = (c * v)[None]
        x0 = v[None].copy() if warm else np.zeros_like(f)
        out.append((pl, rho, c, f, x0))
    return m, dt, out


def random_field(shape, seed=42) -> np.ndarray:
    """Matvec-parity input: U[-1,1] i.i.d."""
    return np.random.default_rng(seed).uniform(-1.0, 1.0, size=shape)


CONFIGS = {
    "C1": dict(kind="mms", nr=16, nt=24, np_=32),
    "C2": dict(kind="conduction", nr=128, nt=128, np_=256),
    "C3": dict(kind="viscosity", nr=256, nt=256, np_=512),
    "C2a": dict(kind="aniso", nr=128, nt=128, np_=256),
    "C2t": dict(kind="tnode", nr=128, nt=128, np_=256),
}


def make(kind: str, **kw) -> Problem:
    return {"mms": mms_problem, "conduction": conduction_problem,
            "viscosity": viscosity_problem, "aniso": aniso_conduction_problem,
            "tnode": tnode_conduction_problem}[kind](**kw)

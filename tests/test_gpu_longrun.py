"""C5 drift check: 200 repeated implicit steps of conduction
(kappa = (T^n)^{5/2} refreshed with mas_op_update every step) followed by
viscosity, warm-started, Delta t frozen at step 0.  GPU (C ABI) vs oracle on
the 40x38x76 downscale (np made even): per-step iteration counts within
max(1, the oracle's own 1-ulp sensitivity) for both solves, rarely different
and with no trend, final T and v within 1e-9 relative L2_V.  The harness arithmetic between solves (kappa = T^{5/2}, rhs =
c T) is done by each side on its own state.
"""
import math

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import workloads as W

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

NSTEPS = 200  # 200 steps on the 40x38x75 downscale (np made even)


@pytest.fixture(scope="module")
def mp():
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    from paper_conf_ipps_caplansl23_b200 import build
    build.build()
    from paper_conf_ipps_caplansl23_b200 import maspcg
    return maspcg


def oracle_trajectory(oracle_mod, oT, L, T0):
    T, v = T0.copy(), L.v0.copy()
    its = []
    for _ in range(NSTEPS):
        kT = T ** 2.5
        f = oT.dirichlet_rhs(kT, (L.c_T * T)[None], L.T_b, None)
        rc, x, itT, _, _ = oT.pcg(kT, L.c_T, f, T[None], L.tol, L.maxit)
        assert rc == oracle_mod.OK
        T = x[0]
        rc, v, itv, _, _ = oT.pcg(L.rho, L.c_v, L.c_v[None] * v, v, L.tol, L.maxit)
        assert rc == oracle_mod.OK
        its.append((itT, itv))
    return T, v, np.array(its)


def test_longrun_drift_vs_oracle(mp, oracle_mod):
    L = W.longrun_problem(40, 38, 76)
    oT = oracle_mod.Oracle(L.mesh, W.DIRICHLET, W.NEUMANN)
    T, v, it_o = oracle_trajectory(oracle_mod, oT, L, L.T0)
    # the oracle's own sensitivity: the same run from T0 perturbed by 1e-16
    # relative -- near the stopping threshold a rounding-level change can move
    # a solve by more than one iteration (R20)
    Tp0 = L.T0 * (1.0 + 1e-16 * np.random.default_rng(3).standard_normal(L.T0.shape))
    _, _, it_p = oracle_trajectory(oracle_mod, oT, L, Tp0)
    env = int(np.abs(it_p - it_o).max())
    # GPU trajectory through the C ABI
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    g = mp.Grid(L.mesh)
    Tg = d(L.T0)[None].contiguous()
    vg = d(L.v0)
    cT, cv, rho, Tb = d(L.c_T), d(L.c_v), d(L.rho), d(L.T_b)
    opT = mp.Operator(g, 1, Tg[0] ** 2.5, cT, W.DIRICHLET, W.NEUMANN)
    opv = mp.Operator(g, 3, rho, cv, W.DIRICHLET, W.NEUMANN)
    it_g = []
    for n in range(NSTEPS):
        if n:
            opT.update((Tg[0] ** 2.5).contiguous(), cT)
        f = (cT * Tg).contiguous()
        opT.dirichlet_rhs(Tb, None, f)
        st, itT, _, _ = opT.solve(f, Tg, L.tol, L.maxit)
        assert st == mp.MAS_OK
        fv = (cv[None] * vg).contiguous()
        st, itv, _, _ = opv.solve(fv, vg, L.tol, L.maxit)
        assert st == mp.MAS_OK
        it_g.append((itT, itv))
    torch.cuda.synchronize()
    dif = np.array(it_g) - it_o
    assert np.abs(dif).max() <= max(1, env), (dif.T, env)
    assert np.abs(dif).mean() <= 0.5
    # no trend: the first and second half differ by at most 1 on average
    h = NSTEPS // 2
    assert abs(dif[:h].mean(0) - dif[h:].mean(0)).max() <= 1.0
    V = oT.volumes()
    rel = lambda a, b: math.sqrt((V * (a - b) ** 2).sum() / (V * b ** 2).sum())
    assert rel(Tg[0].cpu().numpy(), T) <= 1e-9
    assert rel(vg.cpu().numpy(), v) <= 1e-9

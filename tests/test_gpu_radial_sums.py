"""GPU <-> oracle parity of the per-radius array reduction (the paper's
Listings 3-5, "sum0"; reading R27) through the C ABI: device and host
pointers, ragged planes, several components, the C3 plane size, and the
r-slab multi-rank path (virtual ranks: each rank returns its own planes).
Fixed-order sums on both sides in different orders: <= 1e-13 relative to
sum |w x| per plane.
"""
import threading

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import workloads as W

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def mp():
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    from paper_conf_ipps_caplansl23_b200 import build
    build.build()
    from paper_conf_ipps_caplansl23_b200 import maspcg
    return maspcg


def check(got, x, w, ref):
    scale = np.einsum("mijk,jk->mi", np.abs(x), np.abs(w))
    assert np.all(np.abs(got - ref) <= 1e-13 * scale + 1e-300)


@pytest.mark.parametrize("shape,ncomp", [((5, 7, 10), 1), ((9, 13, 70), 3), ((4, 256, 512), 3)])
def test_radial_sums_match_oracle(mp, oracle_mod, shape, ncomp):
    mesh = W.stretched_mesh(*shape)
    rng = np.random.default_rng(11)
    kappa = rng.uniform(0.5, 2.0, size=shape)
    x = rng.standard_normal((ncomp,) + shape)
    w = rng.standard_normal(shape[1:])
    ref = oracle_mod.Oracle(mesh, 0, 1).radial_sums(x, w)
    g = mp.Grid(mesh)
    op = mp.Operator(g, ncomp, torch.from_numpy(kappa).cuda(), None, 0, 1)
    out = torch.empty((ncomp, shape[0]), dtype=torch.float64, device="cuda")
    op.radial_sums(torch.from_numpy(x).cuda(), torch.from_numpy(w).cuda(), out)
    torch.cuda.synchronize()
    check(out.cpu().numpy(), x, w, ref)
    # host pointers (staged), host output (synchronous)
    outh = np.empty((ncomp, shape[0]))
    op.radial_sums(np.ascontiguousarray(x), np.ascontiguousarray(w), outh)
    assert np.array_equal(outh, out.cpu().numpy())


def test_radial_sums_on_r_slabs(mp, oracle_mod):
    shape, P = (11, 8, 16), 3
    mesh = W.stretched_mesh(*shape)
    rng = np.random.default_rng(12)
    x = rng.standard_normal((1,) + shape)
    w = np.zeros(shape[1:])
    w[0] = np.diff(mesh.pF) / (2 * np.pi)  # the north polar-cap phi average
    ref = oracle_mod.Oracle(mesh, 0, 1).radial_sums(x, w)
    vid = mp.virtual_ranks_id(7777)
    res, errs = {}, []

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            with torch.cuda.stream(torch.cuda.Stream()):
                g = mp.Grid(mesh, dist=(P, r, vid))
                sl = slice(g.i0, g.i0 + g.nl)
                op = mp.Operator(g, 1, torch.ones((g.nl,) + shape[1:], dtype=torch.float64,
                                                  device="cuda"), None, 0, 1)
                out = np.empty((1, g.nl))
                op.radial_sums(np.ascontiguousarray(x[:, sl]), w, out)
                res[r] = (g.i0, out)
                op.close()
                g.close()
        except Exception as e:  # noqa: BLE001
            errs.append((r, repr(e)))

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=300)
    assert not errs, errs
    got = np.concatenate([res[r][1] for r in sorted(res, key=lambda q: res[q][0])], axis=1)
    check(got, x, w, ref)

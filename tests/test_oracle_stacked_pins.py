"""Pins for the oracle's stacked PCG (mas_ref_stacked_pcg_solve; NEXT-2,
reading R34 in DESIGN.md §3.9): MAS's viscosity step with each velocity
component at its staggered location -- v_r at r nodes, v_theta at theta nodes
(pole unknowns), v_phi at phi nodes -- solved as ONE Jacobi-PCG on the stacked
vector with the summed V-weighted inner products.  Pinned by what the
mathematics fixes, not by the loop itself:
* one block: the stacked loop is the block's own PCG (mas_ref_*_pcg_solve,
  separately pinned), same iterations and x;
* two identical blocks: every inner product doubles exactly, so alpha, beta
  and the stop decision are those of one block -- x bitwise equal to the
  one-block solve;
* the stacked solution is the dense solve of the block-diagonal system
  (theta nodes in their reduced basis: one unknown per pole and radius);
* the initial residual norm is sqrt(sum_b ||f_b - L_b x0_b||_V^2) (every block
  enters every inner product);
* a block whose rhs and x0 are zero stays exactly zero."""
import math

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import workloads as W

from test_oracle_tnode_pins import reduced, reduced_basis, replicate_poles


def mesh(nr, nt, np_, R=3.0):
    return W.stretched_mesh(nr, nt, np_, 1.0, 2.0, R)


def shape_of(o, pl, om):
    return {om.PLACE_CELL: o.shape, om.PLACE_THETA_NODE: o.tn_shape, om.PLACE_R_NODE: o.rn_shape,
            om.PLACE_PHI_NODE: o.shape}[pl]


def block(om, o, pl, ncomp, seed, zero=False):
    sh = shape_of(o, pl, om)
    rng = np.random.default_rng(seed)
    kappa, c = rng.uniform(0.5, 2.0, size=sh), rng.uniform(0.1, 1.0, size=sh)
    f = rng.standard_normal((ncomp,) + sh)
    if pl == om.PLACE_THETA_NODE:
        c = replicate_poles(c)
        f = replicate_poles(f)
    if zero:
        f = np.zeros_like(f)
    return (o, pl, kappa, c, f, np.zeros_like(f))


def own_pcg(om, blk, tol, maxit):
    o, pl, kappa, c, f, x0 = blk
    fn = {om.PLACE_CELL: o.pcg, om.PLACE_THETA_NODE: o.tn_pcg, om.PLACE_R_NODE: o.rn_pcg,
          om.PLACE_PHI_NODE: o.pn_pcg}[pl]
    return fn(kappa, c, f, x0, tol, maxit)


@pytest.mark.parametrize("pl", [0, 1, 2, 3])
@pytest.mark.parametrize("ncomp", [1, 3])
def test_one_block_is_the_blocks_own_pcg(oracle_mod, pl, ncomp):
    o = oracle_mod.Oracle(mesh(6, 8, 12), 0, 1)
    blk = block(oracle_mod, o, pl, ncomp, 3)
    rc, xs, it, rel, hist = oracle_mod.stacked_pcg([blk], 1e-11, 2000)
    rc1, x1, it1, rel1, hist1 = own_pcg(oracle_mod, blk, 1e-11, 2000)
    assert rc == rc1 == oracle_mod.OK and it == it1
    np.testing.assert_allclose(xs[0], x1, rtol=0, atol=1e-12 * np.abs(x1).max())
    np.testing.assert_allclose(hist, hist1, rtol=1e-11)


def test_two_identical_blocks_reproduce_one_bitwise(oracle_mod):
    o = oracle_mod.Oracle(mesh(5, 6, 16), 0, 1)
    for pl in (oracle_mod.PLACE_R_NODE, oracle_mod.PLACE_THETA_NODE, oracle_mod.PLACE_PHI_NODE):
        blk = block(oracle_mod, o, pl, 1, 7)
        rc1, x1, it1, _, _ = oracle_mod.stacked_pcg([blk], 1e-12, 2000)
        rc2, x2, it2, _, _ = oracle_mod.stacked_pcg([blk, blk], 1e-12, 2000)
        assert rc1 == rc2 == oracle_mod.OK and it1 == it2
        assert np.array_equal(x2[0], x1[0]) and np.array_equal(x2[1], x1[0])


def dense_block(om, o, blk):
    """(A, f, to_reduced, from_reduced) of one block in its own basis."""
    _, pl, kappa, c, f, _ = blk
    sh = shape_of(o, pl, om)
    ap = {om.PLACE_CELL: o.apply, om.PLACE_THETA_NODE: o.tn_apply, om.PLACE_R_NODE: o.rn_apply,
          om.PLACE_PHI_NODE: o.pn_apply}[pl]
    if pl == om.PLACE_THETA_NODE:
        basis = reduced_basis(sh)
        A = np.stack([reduced(ap(kappa, c, e[None])[0], sh) for e in basis], axis=1)
        return A, reduced(f[0], sh), (lambda x: reduced(x[0], sh))
    n = int(np.prod(sh))
    A = np.stack([ap(kappa, c, e.reshape((1,) + sh))[0].ravel() for e in np.eye(n)], axis=1)
    return A, f[0].ravel(), (lambda x: x[0].ravel())


@pytest.mark.parametrize("bcs", [((0, 0), (0, 1), (0, 1)), ((1, 1), (0, 0), (1, 0))])
def test_staggered_stack_is_the_dense_block_solve(oracle_mod, bcs):
    """v_r (r nodes), v_theta (theta nodes), v_phi (phi nodes), each with its
    own boundary conditions, against the dense solve of the block-diagonal
    system; the blocks are scaled differently so that a wrong inner product
    (a block left out, or one block's alpha for all) misses the solution."""
    m = mesh(3, 4, 6)
    blks = []
    for q, (pl, bc) in enumerate(zip((oracle_mod.PLACE_R_NODE, oracle_mod.PLACE_THETA_NODE,
                                      oracle_mod.PLACE_PHI_NODE), bcs)):
        o = oracle_mod.Oracle(m, *bc)
        o_, pl_, kappa, c, f, x0 = block(oracle_mod, o, pl, 1, 20 + q)
        blks.append((o, pl, kappa * 10.0 ** q, c, f * 3.0 ** q, x0))
    rc, xs, it, rel, _ = oracle_mod.stacked_pcg(blks, 1e-14, 2000)
    assert rc == oracle_mod.OK
    for blk, x in zip(blks, xs):
        A, f, red = dense_block(oracle_mod, blk[0], blk)
        xd = np.linalg.solve(A, f)
        assert np.abs(red(x) - xd).max() <= 1e-10 * np.abs(xd).max()


def test_initial_residual_and_zero_block(oracle_mod):
    m = mesh(4, 6, 8)
    o1, o2 = oracle_mod.Oracle(m, 0, 1), oracle_mod.Oracle(m, 0, 0)
    b1 = block(oracle_mod, o1, oracle_mod.PLACE_PHI_NODE, 3, 30)
    b2 = block(oracle_mod, o2, oracle_mod.PLACE_R_NODE, 1, 31)
    rng = np.random.default_rng(32)
    b1 = b1[:5] + (rng.standard_normal(b1[4].shape),)
    b2 = b2[:5] + (rng.standard_normal(b2[4].shape),)
    rc, xs, it, rel, hist = oracle_mod.stacked_pcg([b1, b2], 1e-10, 2000)
    r1 = b1[4] - o1.pn_apply(b1[2], b1[3], b1[5])
    r2 = b2[4] - o2.rn_apply(b2[2], b2[3], b2[5])
    rn0 = math.sqrt((o1.pn_volumes()[None] * r1 * r1).sum() + (o2.rn_volumes()[None] * r2 * r2).sum())
    assert abs(hist[0] - rn0) <= 1e-13 * rn0
    # a zero block next to a live one stays exactly zero
    z = block(oracle_mod, o2, oracle_mod.PLACE_R_NODE, 1, 33, zero=True)
    rc, xs, it, rel, hist = oracle_mod.stacked_pcg([block(oracle_mod, o1, oracle_mod.PLACE_PHI_NODE, 1, 34), z],
                                                   1e-12, 2000)
    assert rc == oracle_mod.OK and it > 0 and not xs[1].any()

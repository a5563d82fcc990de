"""Pins for oracle.bc / oracle.bc_single (Brandes, long double)."""
from fractions import Fraction
from math import comb, factorial, lgamma, log

import numpy as np
import pytest

import gen
import oracle
from brute import bc_pair_dependency, hypercube_delta

INF = 0xFFFFFFFF


def _close(a, b, rel=1e-12):
    return abs(a - b) <= rel * max(1.0, abs(b))


@pytest.mark.parametrize("n,p,seed", [(8, 0.3, 1), (10, 0.25, 2), (12, 0.2, 3), (12, 0.5, 4), (9, 0.15, 5)])
def test_bc_vs_pair_dependency(n, p, seed):
    g = gen.random_simple(n, p, seed)
    for sources in (list(range(n)), [0, 3, 3, 5]):      # duplicates count twice (C14)
        got = oracle.bc(g, sources)
        exp = bc_pair_dependency(g, sources)
        for v in range(n):
            assert _close(got[v], float(exp[v])), (v, got[v], exp[v])


def test_bc_closed_forms_all_sources():
    n = 9
    g = gen.path(n)
    bc = oracle.bc(g, range(n))
    i = np.arange(n)
    assert np.allclose(bc, 2 * i * (n - 1 - i), rtol=0, atol=1e-9)
    n = 8
    bc = oracle.bc(gen.star(n), range(n))
    assert _close(bc[0], (n - 1) * (n - 2)) and np.allclose(bc[1:], 0)
    assert np.allclose(oracle.bc(gen.complete(7), range(7)), 0)
    for n in (5, 7, 9, 11):
        bc = oracle.bc(gen.cycle(n), range(n))
        assert np.allclose(bc, (n - 1) * (n - 3) / 4, rtol=1e-12)
    for d in (2, 3, 4, 5, 6):
        bc = oracle.bc(gen.hypercube(d), range(1 << d))
        assert np.allclose(bc, d * 2 ** (d - 1) - (2 ** d - 1), rtol=1e-12)


def test_hypercube_single_source():
    d = 10
    g = gen.hypercube(d)
    s = 37
    level, sigma, lsig, delta = oracle.bc_single(g, s)
    for v in range(1 << d):
        k = bin(v ^ s).count("1")
        assert level[v] == k
        assert sigma[v] == factorial(k)
        if v != s:
            assert _close(delta[v], float(hypercube_delta(d, k)))


def test_hypercube_sigma_above_2p53():
    d = 20                         # 20! > 2^53: exercises rounding of large counts
    g = gen.hypercube(d)
    level, sigma, lsig, delta = oracle.bc_single(g, 0)
    v = (1 << d) - 1
    assert level[v] == d
    assert _close(sigma[v], float(factorial(d)), rel=1e-15)


def test_lattice_corner_sigma_binomial():
    R, C = 28, 28
    g = gen.grid(R, C)
    level, sigma, lsig, _ = oracle.bc_single(g, 0)
    r, c = np.divmod(np.arange(R * C), C)
    exp = np.array([comb(int(a + b), int(a)) for a, b in zip(r, c)], dtype=np.float64)
    assert np.array_equal(sigma, exp)           # all < 2^53: exact


def test_sigma_beyond_double_range_log2():
    """Full 600x600 grid from the corner: sigma(599,599) = C(1198,599) ~ 2^1193 > DBL_MAX;
    the long-double oracle must still carry it (reading C20)."""
    R = C = 600
    g = gen.grid(R, C)
    level, sigma, lsig, delta = oracle.bc_single(g, 0)
    v = R * C - 1
    exp = (lgamma(1199) - 2 * lgamma(600)) / log(2)
    assert abs(lsig[v] - exp) < 1e-9 * exp
    assert np.isinf(sigma[v])                     # the double view overflows; log2 does not
    assert np.isfinite(delta).all()


def test_dependency_sum_identity_and_leaves():
    """sum_{v != s} delta_s(v) = sum_{t reached, t != s} (d(s,t) - 1) exactly; degree-1
    non-source vertices have delta = 0."""
    g = gen.lattice(60, 80, 0.6, seed=3)
    deg = g.degrees()
    for s in gen.sources(g, 3, stream=6):
        s = int(s)
        level, sigma, lsig, delta = oracle.bc_single(g, s)
        reached = level != INF
        rhs = int((level[reached].astype(np.int64) - 1).sum() + 1)      # t = s contributes -1; undo
        lhs = delta[reached].sum() - delta[s]
        assert abs(lhs - rhs) <= 1e-9 * max(1, rhs)
        leaves = (deg == 1) & reached & (np.arange(g.n) != s)
        assert (delta[leaves] == 0).all()


def test_bc_isolated_source_contributes_zero():
    g = gen.from_edges(6, [0, 1, 2], [1, 2, 3])
    assert np.allclose(oracle.bc(g, [5]), 0)
    assert np.allclose(oracle.bc(g, [0, 5]), oracle.bc(g, [0]))

"""Pins of the f2 oracle (oracle_cg_sr: single-reduction / Chronopoulos-Gear
CG with HPCCG loop control) against things other than itself:

* exact arithmetic -- x0 = 0 makes the first step an exact rational quotient,
  and a plain textbook CG run in Python Fractions (a different algorithm with
  the same exact iterates) fixes the first iterates on a small grid;
* the dense direct solve on the 3x3x3 grid (BJ:north_star);
* an independent numpy textbook CG (same exact iterates: trajectories agree to
  rounding, niters +-1);
* textbook CG invariants (Shewchuk) and the A4 / A11 loop semantics.

A dropped recurrence term (s = w + beta s), a wrong alpha formula or a wrong
lag breaks one of these.  No value here comes from the CUDA path.
"""
import math
from fractions import Fraction

import numpy as np
import pytest

import oracle

from test_oracle_pins import independent_cg, stencil_ref_int


def test_sr_3x3x3_matches_dense_direct_solve():
    p = oracle.generate(3, 3, 3)
    xd = np.linalg.solve(p.to_scipy().toarray(), p.b)
    res = oracle.cg_sr(p, 150, 1e-12)
    assert np.max(np.abs(res["x"] - xd)) < 1e-13
    assert res["niters"] == 5          # same exact iterates as plain CG (A4 lag)
    assert res["normr"] < 1e-13


def test_sr_first_step_exact():
    """x0 = 0: r0 = b, w0 = A b; gamma0 = b.b and delta0 = (Ab).b are exact
    integers, so alpha1 = gamma0/delta0 correctly rounded and x1 = fl(alpha1 b)
    -- the same closed forms as plain CG's first step."""
    for dims, (num, den) in [((3, 3, 3), (6873, 129739)),
                             ((20, 30, 10), (236928, 4056976))]:
        p = oracle.generate(*dims)
        bi = p.b.astype(np.int64)
        assert int(np.dot(bi, stencil_ref_int(*dims, p.b))) == den
        res = oracle.cg_sr(p, 2, 0.0)
        assert res["niters"] == 1
        np.testing.assert_array_equal(res["x"], float(Fraction(num, den)) * p.b)
        assert res["normr"] == math.sqrt(num)


def exact_textbook_cg(A_int, b_int, iters):
    """Plain CG (not the single-reduction form) in exact rational arithmetic."""
    n = len(b_int)
    x = [Fraction(0)] * n
    r = [Fraction(v) for v in b_int]
    p = list(r)
    rr = sum(v * v for v in r)
    out = []
    for _ in range(iters):
        Ap = [sum(A_int[i][j] * p[j] for j in range(n) if A_int[i][j]) for i in range(n)]
        alpha = rr / sum(p[i] * Ap[i] for i in range(n))
        x = [x[i] + alpha * p[i] for i in range(n)]
        r = [r[i] - alpha * Ap[i] for i in range(n)]
        rr_new = sum(v * v for v in r)
        p = [r[i] + (rr_new / rr) * p[i] for i in range(n)]
        rr = rr_new
        out.append(x)
    return out


def test_sr_iterates_equal_exact_rational_cg():
    """The k-th fp64 iterate of the single-reduction oracle equals the k-th
    EXACT iterate of textbook CG to rounding (4x3x3: 36 rows, 6 iterations)."""
    dims = (4, 3, 3)
    p = oracle.generate(*dims)
    A = p.to_scipy().toarray().astype(np.int64).tolist()
    exact = exact_textbook_cg(A, p.b.astype(np.int64).tolist(), 6)
    for k in range(1, 7):
        res = oracle.cg_sr(p, k + 1, 0.0)
        assert res["niters"] == k
        xe = np.array([float(v) for v in exact[k - 1]])
        assert np.max(np.abs(res["x"] - xe)) <= 1e-14 * max(1.0, np.max(np.abs(xe)))


@pytest.mark.parametrize("dims,expect", [((20, 30, 10), 50), ((16, 16, 16), None),
                                         ((31, 17, 9), None)])
def test_sr_vs_independent_textbook_cg(dims, expect):
    """BASELINE.json configs[0] tolerance: niters +-1 of an independent numpy
    CG, x agrees to rounding; 20x30x10 -> 50 iterations."""
    p = oracle.generate(*dims)
    res = oracle.cg_sr(p, 150, 1e-12)
    ni, _, xi = independent_cg(p.to_scipy(), p.b, 150, 1e-12)
    assert abs(res["niters"] - ni) <= 1
    if expect is not None:
        assert res["niters"] == expect
    assert np.max(np.abs(res["x"] - xi)) < 1e-12
    assert oracle.maxabsdiff(res["x"], p.xexact) < 1e-13


def test_sr_trajectory_vs_independent_cg_every_step():
    """Fixed iteration counts (tol 0): the single-reduction iterate tracks the
    textbook iterate to ~1e-13 at every step up to convergence."""
    p = oracle.generate(12, 10, 8)
    A = p.to_scipy()
    for m in [2, 3, 5, 9, 17, 30]:
        xs = oracle.cg_sr(p, m, 0.0)["x"]
        _, _, xi = independent_cg(A, p.b, m, 0.0)
        assert np.max(np.abs(xs - xi)) < 1e-12, m


def test_sr_lagged_normr_and_max_iter_semantics():
    """A4: at most max_iter-1 iterations; normr = ||r|| before the last update."""
    p = oracle.generate(8, 8, 8)
    A = p.to_scipy()
    for m in [2, 3, 6, 10]:
        res = oracle.cg_sr(p, m, 0.0)
        assert res["niters"] == m - 1
        prev = oracle.cg_sr(p, m - 1, 0.0)["x"]
        true_prev = np.linalg.norm(p.b - A @ prev)
        assert abs(res["normr"] - true_prev) <= 1e-12 * np.linalg.norm(p.b)


def test_sr_textbook_invariants():
    """Residuals mutually orthogonal, A-norm error strictly decreasing."""
    p = oracle.generate(7, 6, 5)
    A = p.to_scipy()
    xs = [np.zeros(p.n)] + [oracle.cg_sr(p, k + 1, 0.0)["x"] for k in range(1, 8)]
    rs = [p.b - A @ x for x in xs]
    for i in range(len(rs)):
        for j in range(i):
            c = abs(rs[i] @ rs[j]) / (np.linalg.norm(rs[i]) * np.linalg.norm(rs[j]))
            assert c < 1e-10
    errA = [float((x - 1) @ (A @ (x - 1))) for x in xs]
    assert all(errA[k + 1] < errA[k] for k in range(len(errA) - 1))


def test_sr_degenerate_guard_and_initial_guess():
    """A11: exact convergence with tol 0 stops before 0/0; A5: x0 = solution
    gives gamma0 = 0 -> no iteration."""
    for dims in [(1, 1, 1), (2, 2, 2), (4, 1, 1), (2, 1, 1)]:
        p = oracle.generate(*dims)
        res = oracle.cg_sr(p, 60, 0.0)
        assert np.all(np.isfinite(res["x"]))
        assert oracle.maxabsdiff(res["x"], p.xexact) < 1e-14
        assert res["niters"] < 59
    p = oracle.generate(5, 4, 3)
    res = oracle.cg_sr(p, 50, 1e-12, x0=np.ones(p.n))
    assert res["niters"] == 0 and res["normr"] == 0.0

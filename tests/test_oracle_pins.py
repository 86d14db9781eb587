"""Pins for the CPU oracle (``-m "not gpu"``).

The oracle is only trusted because these tests tie it to things other than
itself: closed forms of the HPCCG operator, exact integer arithmetic, exact
rational arithmetic (``fractions``), a dense direct solve (numpy LAPACK), the
Kronecker-sum spectrum, an independent numpy stencil / CG, and textbook CG
invariants (Shewchuk, cited by the paper as P:L554).  Each test names what a
plausible oracle mistake would break.
"""
import json
import math
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def nnz_closed(nx, ny, nzg):
    # each dimension contributes (3 n - 2) admissible (index, offset) pairs
    return (3 * nx - 2) * (3 * ny - 2) * (3 * nzg - 2)


def stencil_ref_int(nx, ny, nzg, x):
    """Independent numpy form of y = A x for integer x: A = 28 I - K, K the
    truncated 3x3x3 box sum (A6).  int64, exact."""
    g = x.reshape(nzg, ny, nx).astype(np.int64)
    pad = np.pad(g, 1)
    box = np.zeros_like(g)
    for dz in range(3):
        for dy in range(3):
            for dx in range(3):
                box += pad[dz:dz + nzg, dy:dy + ny, dx:dx + nx]
    return (28 * g - box).reshape(-1)


# --------------------------------------------------------------- generate

@pytest.mark.parametrize("dims", [(1, 1, 1), (2, 2, 2), (3, 3, 3), (4, 1, 1),
                                  (20, 30, 10), (7, 5, 6)])
def test_generate_nnz_closed_form(dims):
    """nnz = prod_d (3 n_d - 2): a dropped/extra boundary neighbour fails."""
    p = oracle.generate(*dims)
    assert p.nnz == nnz_closed(*dims)


def test_generate_slabs_match_global_rows():
    """Chimney decomposition: slab r holds exactly rows [r n, (r+1) n) of the
    global problem, with the per-rank nnz closed form."""
    nx, ny, nz, P = 5, 7, 3, 4
    g = oracle.generate(nx, ny, nz * P)
    n = nx * ny * nz
    assert g.nnz == nnz_closed(nx, ny, nz * P)
    for r in range(P):
        s = oracle.generate(nx, ny, nz, r, P)
        lo, hi = g.row_ptr[r * n], g.row_ptr[(r + 1) * n]
        np.testing.assert_array_equal(s.row_ptr, g.row_ptr[r * n:(r + 1) * n + 1] - lo)
        np.testing.assert_array_equal(s.cols, g.cols[lo:hi])
        np.testing.assert_array_equal(s.vals, g.vals[lo:hi])
        np.testing.assert_array_equal(s.b, g.b[r * n:(r + 1) * n])
        exp = (3 * nx - 2) * (3 * ny - 2) * (3 * nz - (r == 0) - (r == P - 1))
        assert s.nnz == exp


def test_generate_interior_rows_and_b():
    """Interior rows: diag 27 and 26 x (-1), row sum 1; b = A.1 (row sums);
    b_i = 28 - nnz_i; columns strictly ascending (A8 canonical order)."""
    p = oracle.generate(6, 5, 4)
    A = p.to_scipy().toarray()
    for i in range(p.n):
        c = p.cols[p.row_ptr[i]:p.row_ptr[i + 1]]
        assert np.all(np.diff(c) > 0)
        nnz_i = len(c)
        assert A[i, i] == 27.0
        assert p.b[i] == 28 - nnz_i
    np.testing.assert_array_equal(A.sum(axis=1), p.b)
    iz, iy, ix = 2, 2, 2
    i = iz * 30 + iy * 6 + ix
    row = A[i]
    assert (row != 0).sum() == 27 and row.sum() == 1.0
    assert sorted(row[row != 0].tolist()) == [-1.0] * 26 + [27.0]
    assert np.all(p.x == 0.0) and np.all(p.xexact == 1.0)


def test_generate_symmetric_and_kronecker_form():
    """A == A^T exactly and A == 28 I - T_z (x) T_y (x) T_x with T =
    tridiag(1,1,1): a transposed / shifted index fails."""
    nx, ny, nz = 4, 3, 5
    A = oracle.generate(nx, ny, nz).to_scipy().toarray()
    np.testing.assert_array_equal(A, A.T)

    def T(n):
        return np.eye(n) + np.eye(n, k=1) + np.eye(n, k=-1)
    K = np.kron(np.kron(T(nz), T(ny)), T(nx))
    np.testing.assert_array_equal(A, 28.0 * np.eye(nx * ny * nz) - K)


def test_generate_spectrum_closed_form():
    """lambda = 28 - prod_d (1 + 2 cos(k_d pi / (n_d + 1))): SPD, kappa < 37."""
    nx, ny, nz = 4, 3, 5
    A = oracle.generate(nx, ny, nz).to_scipy().toarray()
    ev = np.linalg.eigvalsh(A)
    lam = []
    for kz in range(1, nz + 1):
        for ky in range(1, ny + 1):
            for kx in range(1, nx + 1):
                lam.append(28 - (1 + 2 * math.cos(kx * math.pi / (nx + 1)))
                           * (1 + 2 * math.cos(ky * math.pi / (ny + 1)))
                           * (1 + 2 * math.cos(kz * math.pi / (nz + 1))))
    np.testing.assert_allclose(np.sort(ev), np.sort(lam), atol=1e-11)
    assert ev.min() > 1.0 and ev.max() < 37.0


def test_b_sum_and_norm_closed_forms():
    """sum b = 28 N - nnz; b.b = 784 N - 56 nnz + prod_d (9 n_d - 10)
    (20x30x10: 25,088 and 236,928)."""
    for dims in [(20, 30, 10), (3, 3, 3), (9, 4, 7)]:
        p = oracle.generate(*dims)
        N, nnz = p.n, p.nnz
        assert p.b.sum() == 28 * N - nnz
        prod = 1
        for d in dims:
            prod *= 9 * d - 10
        assert oracle.ddot(p.b, p.b) == 784 * N - 56 * nnz + prod
    p = oracle.generate(20, 30, 10)
    assert p.b.sum() == 25088 and oracle.ddot(p.b, p.b) == 236928


# ------------------------------------------------------------------ spmv

def test_spmv_A_ones_is_b_bitwise():
    p = oracle.generate(20, 30, 10)
    y = oracle.spmv(p, np.ones(p.n))
    np.testing.assert_array_equal(y, p.b)


@pytest.mark.parametrize("dims", [(20, 30, 10), (1, 1, 1), (4, 1, 1), (2, 3, 1), (33, 2, 5)])
def test_spmv_integer_vectors_exact(dims):
    """Integer x: every order gives the exact result, so this pins all the
    indexing against an independent 3-D stencil."""
    p = oracle.generate(*dims)
    x = synth.integers(p.n, 7, -1000, 1000)
    y = oracle.spmv(p, x)
    np.testing.assert_array_equal(y.astype(np.int64), stencil_ref_int(*dims, x))


def test_spmv_symmetry_integer():
    p = oracle.generate(9, 8, 7)
    u = synth.integers(p.n, 1, -50, 50)
    v = synth.integers(p.n, 2, -50, 50)
    Au, Av = oracle.spmv(p, u), oracle.spmv(p, v)
    assert int(np.dot(u.astype(np.int64), Av.astype(np.int64))) == \
        int(np.dot(Au.astype(np.int64), v.astype(np.int64)))


def test_spmv_real_error_bound():
    """Real x: |y - exact| <= 27 eps sum_j |a_ij x_j| (exact via Fractions)."""
    p = oracle.generate(6, 5, 4)
    x = synth.uniform(p.n, 11)
    y = oracle.spmv(p, x)
    eps = 2.0 ** -53
    for i in range(p.n):
        lo, hi = p.row_ptr[i], p.row_ptr[i + 1]
        ex = sum(Fraction(p.vals[k]) * Fraction(x[p.cols[k]]) for k in range(lo, hi))
        mag = sum(abs(p.vals[k] * x[p.cols[k]]) for k in range(lo, hi))
        assert abs(Fraction(y[i]) - ex) <= Fraction(27 * eps * mag)


def test_spmv_slab_halo_layout():
    """Slab rows with the [lower halo | n owned | upper halo] x layout give
    the same bits as the global rows (col_offset = r n - plane)."""
    nx, ny, nz, P = 6, 5, 3, 3
    g = oracle.generate(nx, ny, nz * P)
    xg = synth.uniform(g.n, 5)
    yg = oracle.spmv(g, xg)
    n, plane = nx * ny * nz, nx * ny
    for r in range(P):
        s = oracle.generate(nx, ny, nz, r, P)
        xl = np.zeros(n + 2 * plane)
        lo = r * n - plane
        for j in range(n + 2 * plane):
            if 0 <= lo + j < g.n:
                xl[j] = xg[lo + j]
        np.testing.assert_array_equal(oracle.spmv(s, xl), yg[r * n:(r + 1) * n])
    rows = synth.sample_rows(g.n, 20, 3)
    np.testing.assert_array_equal(oracle.spmv_rows(nx, ny, nz * P, rows, xg), yg[rows])


# ------------------------------------------------------------------ ddot

def test_ddot_jacc_integer_inputs_exact():
    """Fig. 2 recipe: integer inputs 0..100 -> exact int64 sum."""
    cfg = json.load(open(os.path.join(GOLDEN, "paper_inputs.json")))["fig2_blas1"]
    n = cfg["size"]
    x, y = synth.jacc_vector(n, 42), synth.jacc_vector(n, 43)
    assert x.min() >= 0 and x.max() <= cfg["value_scale"] and np.all(x == np.rint(x))
    exact = int(np.dot(x.astype(np.int64), y.astype(np.int64)))
    assert oracle.ddot(x, y) == float(exact)


def test_ddot_compensated_vs_exact_rational():
    x, y = synth.uniform(3000, 1), synth.uniform(3000, 2)
    ex = sum(Fraction(a) * Fraction(b) for a, b in zip(x, y))
    got = oracle.ddot(x, y)
    assert abs(Fraction(got) - ex) <= abs(ex) * Fraction(2.0 ** -52)


def test_ddot_compensation_present():
    """Naive summation gives 0 here; Dot2 must give the exact 1."""
    x = np.array([1e16, 1.0, -1e16])
    assert oracle.ddot(x, np.ones(3)) == 1.0
    # spans more than one 2^16 chunk: the chunk combination is compensated too
    n = 3 * 65536
    x = np.zeros(n)
    x[0], x[70000], x[140000] = 1e16, 1.0, -1e16
    assert oracle.ddot(x, np.ones(n)) == 1.0
    assert oracle.ddot(np.zeros(0), np.zeros(0)) == 0.0


def test_ddot_thread_count_independent():
    x, y = synth.uniform(300001, 3), synth.uniform(300001, 4)
    t0 = oracle.get_threads()
    oracle.set_threads(1)
    a = oracle.ddot(x, y)
    oracle.set_threads(max(t0, 2))
    b = oracle.ddot(x, y)
    oracle.set_threads(t0)
    assert a == b


# ---------------------------------------------------------------- waxpby

def test_waxpby_jacc_axpy_exact():
    """JACC AXPY x += 2.5 y (Fig. 2) on integer inputs is
    exact (multiples of 0.5)."""
    n = 100000
    x, y = synth.jacc_vector(n, 42), synth.jacc_vector(n, 43)
    w = oracle.waxpby(1.0, x, 2.5, y)
    exact = (2 * x.astype(np.int64) + 5 * y.astype(np.int64))
    np.testing.assert_array_equal(w * 2, exact.astype(np.float64))
    xx = x.copy()
    oracle.waxpby(1.0, xx, 2.5, y, out=xx)   # in-place alias
    np.testing.assert_array_equal(xx, w)


@pytest.mark.parametrize("alpha,beta", [(1.0, 0.37), (0.61, 1.0), (0.3, -0.7), (1.0, 0.0)])
def test_waxpby_canonical_rounding(alpha, beta):
    """Canonical forms (A10), checked with exact rationals: alpha==1 ->
    round(x + beta y); beta==1 -> round(alpha x + y); else
    round(alpha x + round(beta y))."""
    x, y = synth.uniform(500, 8), synth.uniform(500, 9)
    w = oracle.waxpby(alpha, x, beta, y)
    for i in range(500):
        if alpha == 1.0:
            ex = Fraction(x[i]) + Fraction(beta) * Fraction(y[i])
        elif beta == 1.0:
            ex = Fraction(alpha) * Fraction(x[i]) + Fraction(y[i])
        else:
            ex = Fraction(alpha) * Fraction(x[i]) + Fraction(beta * y[i])
        assert w[i] == float(ex)


# -------------------------------------------------------------------- CG

def test_cg_3x3x3_matches_dense_direct_solve():
    """BJ:north_star: a dense direct solve on a 3x3x3 grid must agree."""
    p = oracle.generate(3, 3, 3)
    A = p.to_scipy().toarray()
    xd = np.linalg.solve(A, p.b)
    assert np.max(np.abs(xd - 1.0)) < 1e-14
    res = oracle.cg(p, 150, 1e-12)
    assert np.max(np.abs(res["x"] - xd)) < 1e-13
    # b excites 4 eigenvalues -> r_4 ~ 0; lagged check -> niters = 5 (A4)
    assert res["niters"] == 5
    assert res["normr"] < 1e-13


def test_cg_first_step_exact():
    """x0 = 0: r0 = p1 = b, rtrans = b.b and p.Ap = b.Ab are exact integers,
    so alpha1 is the correctly rounded quotient and x1 = fl(alpha1 b)."""
    for dims, (num, den) in [((3, 3, 3), (6873, 129739)),
                             ((20, 30, 10), (236928, 4056976))]:
        p = oracle.generate(*dims)
        bi = p.b.astype(np.int64)
        Ab = stencil_ref_int(*dims, p.b)
        assert int(np.dot(bi, bi)) == num and int(np.dot(bi, Ab)) == den
        alpha = float(Fraction(num, den))
        res = oracle.cg(p, 2, 0.0)
        assert res["niters"] == 1
        np.testing.assert_array_equal(res["x"], alpha * p.b)
        assert res["normr"] == math.sqrt(num)


def test_cg_iterates_equal_exact_rational_cg():
    """The k-th fp64 iterate of oracle_cg equals the k-th EXACT iterate of
    textbook CG (Python Fractions, 4x3x3 grid, k <= 6) to rounding: pins the
    trajectory beyond the first step, not just the end point."""
    from test_oracle_sr_pins import exact_textbook_cg
    p = oracle.generate(4, 3, 3)
    A = p.to_scipy().toarray().astype(np.int64).tolist()
    exact = exact_textbook_cg(A, p.b.astype(np.int64).tolist(), 6)
    for k in range(1, 7):
        res = oracle.cg(p, k + 1, 0.0)
        assert res["niters"] == k
        xe = np.array([float(v) for v in exact[k - 1]])
        assert np.max(np.abs(res["x"] - xe)) <= 1e-14 * max(1.0, np.max(np.abs(xe)))


def independent_cg(A, b, max_iter, tol):
    """Textbook CG written independently (numpy dot, HPCCG loop control)."""
    x = np.zeros_like(b)
    r = b - A @ x
    p = r.copy()
    rtrans = float(r @ r)
    normr = math.sqrt(rtrans)
    k, niters = 1, 0
    while k < max_iter and normr > tol:
        if k > 1:
            old, rtrans = rtrans, float(r @ r)
            p = r + (rtrans / old) * p
        normr = math.sqrt(rtrans)
        Ap = A @ p
        alpha = rtrans / float(p @ Ap)
        x = x + alpha * p
        r = r - alpha * Ap
        niters = k
        k += 1
    return niters, normr, x


@pytest.mark.parametrize("dims,expect", [((20, 30, 10), 50), ((3, 3, 3), 5), ((16, 16, 16), None)])
def test_cg_iteration_count_vs_independent_cg(dims, expect):
    """BASELINE.json configs[0]: tol 1e-12, max_iter 150.  Independent numpy
    CG agrees on niters (+-1) and x; SURVEY's two scratch implementations
    give 50 for 20x30x10."""
    p = oracle.generate(*dims)
    res = oracle.cg(p, 150, 1e-12)
    ni, nr, xi = independent_cg(p.to_scipy(), p.b, 150, 1e-12)
    assert abs(res["niters"] - ni) <= 1
    if expect is not None:
        assert res["niters"] == expect
    assert np.max(np.abs(res["x"] - xi)) < 1e-12
    assert oracle.maxabsdiff(res["x"], p.xexact) < 1e-13
    assert res["normr"] <= 1e-12 and res["normr"] > 0


def test_cg_lagged_normr_and_max_iter_semantics():
    """A4: at most max_iter-1 iterations; the returned normr is ||r|| of the
    iterate BEFORE the last update (lagged), i.e. the true residual of the
    run with one iteration fewer."""
    p = oracle.generate(8, 8, 8)
    A = p.to_scipy()
    for m in [2, 3, 6, 10]:
        res = oracle.cg(p, m, 0.0)
        assert res["niters"] == m - 1
        prev = oracle.cg(p, m - 1, 0.0)["x"]
        true_prev = np.linalg.norm(p.b - A @ prev)
        assert abs(res["normr"] - true_prev) <= 1e-12 * np.linalg.norm(p.b)
        cur = np.linalg.norm(p.b - A @ res["x"])
        assert cur < res["normr"]     # CG residual decreased past normr


def test_cg_textbook_invariants():
    """Residuals mutually orthogonal, A-norm error strictly decreasing
    (Shewchuk).  A wrong sign/index in alpha or beta breaks these."""
    p = oracle.generate(7, 6, 5)
    A = p.to_scipy()
    xs = [np.zeros(p.n)] + [oracle.cg(p, k + 1, 0.0)["x"] for k in range(1, 8)]
    rs = [p.b - A @ x for x in xs]
    for i in range(len(rs)):
        for j in range(i):
            c = abs(rs[i] @ rs[j]) / (np.linalg.norm(rs[i]) * np.linalg.norm(rs[j]))
            assert c < 1e-10
    errA = [float((x - 1) @ (A @ (x - 1))) for x in xs]
    assert all(errA[k + 1] < errA[k] for k in range(len(errA) - 1))


def test_cg_degenerate_exact_convergence_guard():
    """A11: tiny grids reach r == 0 exactly with tol = 0; the guard stops
    before 0/0 so x stays finite and exact-ish."""
    for dims in [(1, 1, 1), (2, 2, 2), (4, 1, 1), (2, 1, 1)]:
        p = oracle.generate(*dims)
        res = oracle.cg(p, 60, 0.0)
        assert np.all(np.isfinite(res["x"]))
        assert oracle.maxabsdiff(res["x"], p.xexact) < 1e-14
        assert res["niters"] < 59


def test_cg_nonzero_initial_guess():
    """A5: x is in/out; starting at the solution gives r0 = 0 -> no iteration."""
    p = oracle.generate(5, 4, 3)
    res = oracle.cg(p, 50, 1e-12, x0=np.ones(p.n))
    assert res["niters"] == 0 and res["normr"] == 0.0
    np.testing.assert_array_equal(res["x"], np.ones(p.n))


# ------------------------------------------------ f3: JACC 2-D AXPY / DOT

def test_2d_axpy_dot_fig2_inputs_exact():
    """Fig. 2's multidimensional example: SIZE = 1000,
    round(rand*100) inputs, alpha = 2.5 -> AXPY and DOT exact."""
    cfg = json.load(open(os.path.join(GOLDEN, "paper_inputs.json")))["fig2_blas1_2d"]
    m = n = cfg["size"]
    x, y = synth.jacc_vector(m * n, 42), synth.jacc_vector(m * n, 43)
    w = oracle.waxpby2d(m, n, m, 1.0, x, 2.5, y)
    np.testing.assert_array_equal(2 * w, (2 * x + 5 * y))
    assert oracle.ddot2d(m, n, m, x, y) == float(int(np.dot(x.astype(np.int64), y.astype(np.int64))))


def test_2d_leading_dimension_semantics():
    """Only the m x n block of an ld x n column-major array is touched; the
    result equals the 1-D routines on that block (numpy column-major slice)."""
    m, n, ld = 37, 23, 50
    x, y = synth.uniform(ld * n, 1), synth.uniform(ld * n, 2)
    w = oracle.waxpby2d(m, n, ld, 0.3, x, -0.7, y)
    X = x.reshape(n, ld).T
    Y = y.reshape(n, ld).T
    W = w.reshape(n, ld).T
    np.testing.assert_array_equal(W[m:, :], X[m:, :])          # padding untouched
    blk = oracle.waxpby(0.3, np.ascontiguousarray(X[:m, :].T).ravel(), -0.7,
                        np.ascontiguousarray(Y[:m, :].T).ravel())
    np.testing.assert_array_equal(np.ascontiguousarray(W[:m, :].T).ravel(), blk)
    ex = sum(Fraction(a) * Fraction(b) for a, b in zip(X[:m, :].ravel(), Y[:m, :].ravel()))
    got = oracle.ddot2d(m, n, ld, x, y)
    assert abs(Fraction(got) - ex) <= abs(ex) * Fraction(2.0 ** -52)


# ------------------------------------------------------------- a.9 verify

def _maxabsdiff_exact(x, xe):
    """Independent definition: for each i the EXACT difference as a rational,
    rounded once to the nearest double (= what one IEEE subtraction returns),
    then the largest magnitude; entries whose difference is NaN are skipped
    (HPCCG's `if (diff > max)` never takes a NaN, reading A26)."""
    best = Fraction(0)
    for a, b in zip(x.tolist(), xe.tolist()):
        if math.isnan(a) or math.isnan(b):
            continue
        d = abs(Fraction(float(np.float64(a))) - Fraction(float(np.float64(b))))
        d = Fraction(float(d))                      # one correctly rounded subtraction
        best = max(best, d)
    return float(best)


@pytest.mark.parametrize("pos", ["first", "middle", "last"])
@pytest.mark.parametrize("sign", [1.0, -1.0])
def test_maxabsdiff_planted_spike_closed_form(pos, sign):
    """a.9 (HPCCG compute_residual; BJ:north_star "final max|x-1|"): x = 1 +
    noise (|noise| < 2^-10) with ONE planted deviation d = sign * 0.75 -- the
    result is exactly 0.75 (1 +- 0.75 and its difference with 1 are exact).
    Breaks: a dropped fabs (sign -1), a loop that skips the first / last
    element, a min instead of a max, a constant return."""
    n = 4099
    x = 1.0 + synth.uniform(n, 91, -2.0 ** -10, 2.0 ** -10)
    j = {"first": 0, "middle": n // 2, "last": n - 1}[pos]
    x[j] = 1.0 + sign * 0.75
    xe = np.ones(n)
    assert oracle.maxabsdiff(x, xe) == 0.75
    assert oracle.maxabsdiff(x, xe) == np.max(np.abs(x - xe))


def test_maxabsdiff_vs_exact_rational_general_xexact():
    """Arbitrary x and x_exact (not only x_exact = 1): equal to the exact
    rational definition above, bit for bit; both signs of the largest
    deviation are exercised by the two seeds."""
    for seed in (5, 6, 7):
        x = synth.uniform(1537, seed, -3.0, 3.0)
        xe = synth.uniform(1537, seed + 100, -3.0, 3.0)
        assert oracle.maxabsdiff(x, xe) == _maxabsdiff_exact(x, xe)


def test_maxabsdiff_zero_signed_zero_and_subnormals():
    """x == x_exact -> exactly +0 (also with -0 against +0); a single
    subnormal deviation is returned, not flushed to zero (either sign)."""
    n = 257
    xe = np.zeros(n)
    x = np.zeros(n)
    x[::2] = -0.0
    r = oracle.maxabsdiff(x, xe)
    assert r == 0.0 and not math.copysign(1.0, r) < 0
    tiny = 5e-324
    for j, s in ((0, 1.0), (n - 1, -1.0), (100, -1.0)):
        y = x.copy()
        y[j] = s * tiny
        assert oracle.maxabsdiff(y, xe) == tiny
    ones = np.ones(n)
    assert oracle.maxabsdiff(ones, ones) == 0.0
    assert oracle.maxabsdiff(np.ones(0), np.ones(0)) == 0.0


def test_maxabsdiff_nan_entries_skipped():
    """Reading A26: a NaN entry compares false against the running maximum
    (HPCCG's `if (diff > max)`), so it is skipped; the finite entries still
    decide the result."""
    x = np.ones(64)
    x[3] = np.nan
    x[40] = 1.5
    assert oracle.maxabsdiff(x, np.ones(64)) == 0.5 == _maxabsdiff_exact(x, np.ones(64))

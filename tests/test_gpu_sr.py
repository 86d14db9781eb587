"""GPU parity tests for SURVEY f2, the single-reduction (Chronopoulos-Gear)
CG (HPCCG_OPT_CG_VARIANT = 1), against its oracle (oracle.cg_sr, pinned in
tests/test_oracle_sr_pins.py) and against HPCCG's CG oracle.

Bars as for HPCCG's CG (BASELINE.json north_star): niters +-1, final x /
max|x-1| / normr within 1e-10; the first step bitwise (exact integers);
every launch mode (while-graph with any unroll, per-iteration graph, plain,
timed, any vector unroll) bit-identical to each other.
"""
import numpy as np
import pytest

import oracle
import synth  # noqa: F401  (seeded generators; CG inputs are generated)

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H  # noqa: E402

CG_ATOL = 1e-10


@pytest.fixture(scope="module")
def ctx():
    c = H.Context(0)
    yield c
    c.close()


def sr(p):
    p.set_option(H.HPCCG_OPT_CG_VARIANT, 1)
    return p


def check(res, p, oref, ref):
    assert abs(res["niters"] - oref["niters"]) <= 1, (res["niters"], oref["niters"])
    assert abs(p.maxabsdiff() - oracle.maxabsdiff(oref["x"], ref.xexact)) <= CG_ATOL
    assert abs(res["normr"] - oref["normr"]) <= CG_ATOL
    assert np.max(np.abs(p.get_vec(H.HPCCG_VEC_X) - oref["x"])) <= CG_ATOL


@pytest.mark.parametrize("persist", [0, 1])
@pytest.mark.parametrize("dims", [(20, 30, 10), (3, 3, 3), (16, 16, 16), (33, 9, 3), (31, 17, 9),
                                  (64, 32, 40)])
def test_sr_cg_vs_oracle(ctx, dims, persist):
    """persist 0: the while-graph of 2-kernel iterations; persist 1: problems
    that fit one cluster's shared memory run the on-chip single-reduction
    kernel (2 cluster barriers per iteration), larger ones the while-graph."""
    with H.Problem(ctx, *dims) as p:
        sr(p)
        p.set_option(H.HPCCG_OPT_PERSISTENT, persist)
        ref = oracle.generate(*dims)
        oref = oracle.cg_sr(ref, 150, 1e-12)
        res = p.solve(150, 1e-12)
        n = dims[0] * dims[1] * dims[2]
        assert p.stats()["graph_mode"] == (5 if persist and n <= 9000 else 2)
        check(res, p, oref, ref)
        # same solution as HPCCG's CG
        assert abs(res["niters"] - oracle.cg(ref, 150, 1e-12)["niters"]) <= 1
        if dims == (20, 30, 10):
            assert res["niters"] == 50


@pytest.mark.parametrize("persist", [0, 1])
def test_sr_first_step_exact(ctx, persist):
    """x0 = 0: gamma0 = b.b, delta0 = (Ab).b exact integers -> alpha1 correctly
    rounded, x1 = fl(alpha1 b) bitwise, normr = sqrt(b.b)."""
    with H.Problem(ctx, 20, 30, 10) as p:
        sr(p)
        p.set_option(H.HPCCG_OPT_PERSISTENT, persist)
        r = p.solve(2, 0.0)
        assert r["niters"] == 1
        b = p.get_vec(H.HPCCG_VEC_B)
        np.testing.assert_array_equal(p.get_vec(H.HPCCG_VEC_X), (236928 / 4056976) * b)
        assert r["normr"] == np.sqrt(236928.0)


@pytest.mark.parametrize("rows", [1, 2])
def test_sr_launch_modes_bitwise_identical(ctx, rows):
    """While-graph (unroll 1 -> 2, 3 -> 4, 4, 6), per-iteration graph (pairs of
    iterations + host poll), plain and timed launches, vector unroll 1/2/4:
    the same arithmetic in the same order -> identical bits."""
    dims = (24, 20, 12)
    outs, xs = [], []
    with H.Problem(ctx, *dims) as p:
        sr(p)
        p.set_option(H.HPCCG_OPT_PERSISTENT, 0)
        p.set_option(H.HPCCG_OPT_SPMV_ROWS, rows)
        cfgs = [dict(wu=4), dict(wu=1), dict(wu=3), dict(wu=6), dict(wh=0), dict(graph=0),
                dict(timing=1), dict(unroll=1), dict(unroll=2), dict(pdl=0)]
        for c in cfgs:
            p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n))
            p.set_option(H.HPCCG_OPT_WHILE_UNROLL, c.get("wu", 4))
            p.set_option(H.HPCCG_OPT_WHILE, c.get("wh", 1))
            p.set_option(H.HPCCG_OPT_GRAPH, c.get("graph", 1))
            p.set_option(H.HPCCG_OPT_TIMING, c.get("timing", 0))
            p.set_option(H.HPCCG_OPT_VEC_UNROLL, c.get("unroll", 4))
            p.set_option(H.HPCCG_OPT_PDL, c.get("pdl", 1))
            r = p.solve(150, 1e-12)
            outs.append((r["niters"], r["normr"]))
            xs.append(p.get_vec(H.HPCCG_VEC_X))
            st = p.stats()
            assert st["spmv_launches"] == r["niters"] + 2
            if c.get("timing"):
                assert st["spmv_ms"] > 0 and st["update_ms"] > 0 and st["pupdate_ms"] == 0
    for o, x in zip(outs[1:], xs[1:]):
        assert o == outs[0]
        np.testing.assert_array_equal(x, xs[0])


@pytest.mark.parametrize("wh,persist", [(0, 0), (1, 0), (1, 1)])
def test_sr_max_iter_semantics_odd_and_even(ctx, wh, persist):
    """A4 with the parity-double-buffered loop state: at most max_iter - 1
    iterations for odd and even counts, in the while-graph, in the
    per-iteration graph (which replays iteration PAIRS) and on chip."""
    with H.Problem(ctx, 8, 8, 8) as p:
        sr(p)
        p.set_option(H.HPCCG_OPT_PERSISTENT, persist)
        p.set_option(H.HPCCG_OPT_WHILE, wh)
        ref = oracle.generate(8, 8, 8)
        for m in [1, 2, 3, 4, 10, 37]:
            p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n))
            r = p.solve(m, 0.0)
            o = oracle.cg_sr(ref, m, 0.0)
            assert r["niters"] == o["niters"] == m - 1
            assert abs(r["normr"] - o["normr"]) <= CG_ATOL
            assert np.max(np.abs(p.get_vec(H.HPCCG_VEC_X) - o["x"])) <= CG_ATOL
        p.set_vec(H.HPCCG_VEC_X, np.ones(p.n))       # start at the solution
        r = p.solve(50, 1e-12)
        assert r["niters"] == 0 and r["normr"] == 0.0


@pytest.mark.parametrize("wh", [0, 1])
def test_sr_tolerance_stop(ctx, wh):
    with H.Problem(ctx, 20, 30, 10) as p:
        sr(p)
        p.set_option(H.HPCCG_OPT_PERSISTENT, 0)
        p.set_option(H.HPCCG_OPT_WHILE, wh)
        r = p.solve(150, 1e-12)
        assert r["niters"] == 50
        assert p.stats()["graph_mode"] == (2 if wh else 1)
        assert p.solve(150, 1e-12)["niters"] <= 2


@pytest.mark.parametrize("persist", [0, 1])
@pytest.mark.parametrize("dims", [(1, 1, 1), (2, 2, 2), (4, 1, 1)])
def test_sr_degenerate_guard(ctx, dims, persist):
    with H.Problem(ctx, *dims) as p:
        sr(p)
        p.set_option(H.HPCCG_OPT_PERSISTENT, persist)
        r = p.solve(60, 0.0)
        assert np.all(np.isfinite(p.get_vec(H.HPCCG_VEC_X))) and p.maxabsdiff() < 1e-14
        assert r["niters"] < 59


@pytest.mark.parametrize("P", [2, 3, 4])
def test_sr_loopback_matches_global_oracle(P):
    """z-slabs: one allreduce of (gamma, delta) per iteration reproduces the
    global single-reduction CG (niters +-1, 1e-10)."""
    nx, ny, nz = 16, 12, 6
    with H.Context(0, nranks=P, loopback=True) as c, H.Problem(c, nx, ny, nz) as p:
        sr(p)
        ref = oracle.generate(nx, ny, nz * P)
        oref = oracle.cg_sr(ref, 150, 1e-12)
        res = p.solve(150, 1e-12)
        check(res, p, oref, ref)


def test_sr_nccl_one_rank_code_path():
    """1-rank NCCL communicator: halo exchange on the comm stream, the
    per-slab (gamma, delta) finisher and ONE ncclAllReduce of 2 doubles per
    iteration inside the captured (paired) per-iteration graph."""
    dims = (16, 12, 6)
    uid = H.hpccg_unique_id()
    with H.Context(0, rank=0, nranks=1, unique_id=uid) as c, H.Problem(c, *dims) as p:
        sr(p)
        ref = oracle.generate(*dims)
        oref = oracle.cg_sr(ref, 150, 1e-12)
        for timing in (0, 1):
            p.set_option(H.HPCCG_OPT_TIMING, timing)
            p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n))
            res = p.solve(150, 1e-12)
            assert p.stats()["graph_mode"] == (0 if timing else 1)
            check(res, p, oref, ref)


@pytest.mark.parametrize("rows", [2, 1])
def test_sr_full_128cubed(ctx, rows):
    """BASELINE configs[1] size: to tol 1e-12 vs the full oracle (rows = 1
    gives 8192 SpMV blocks > 4096: the one-block (gamma, delta) finisher path);
    the bench's 500-iteration tol-0 run stays at the solution."""
    with H.Problem(ctx, 128, 128, 128) as p:
        sr(p)
        p.set_option(H.HPCCG_OPT_SPMV_ROWS, rows)
        ref = oracle.generate(128, 128, 128)
        oref = oracle.cg_sr(ref, 150, 1e-12)
        res = p.solve(150, 1e-12)
        check(res, p, oref, ref)
        p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n))
        r500 = p.solve(501, 0.0)
        assert r500["niters"] == 500
        assert p.maxabsdiff() < 1e-13 and 0 <= r500["normr"] < 1e-40


@pytest.mark.parametrize("dims,max_iter,tol", [((20, 30, 10), 150, 1e-12), ((31, 17, 9), 40, 0.0),
                                               ((64, 48, 40), 18, 0.0), ((64, 48, 40), 17, 0.0),
                                               ((33, 9, 3), 7, 0.0), ((16, 16, 16), 150, 1e-12)])
def test_sr_ring_deferred_x_bitwise(ctx, dims, max_iter, tol):
    """f2 with x deferred over m iterations (HPCCG_OPT_DEFER_X = m): p_k goes
    to ring slot k % (m + 1), the update with k % m == 0 also applies x =
    fma(alpha_j, p_j, x) for the last m directions (p_k from registers), and
    cg_xfix_ring_kernel the pending ones after the loop -- the FMAs of the
    undeferred update in the same order, so niters, normr and x are bit for
    bit equal, in every launch mode; iteration counts ending 0..m-1 after a
    flush; odd n."""
    with H.Problem(ctx, *dims) as p:
        sr(p)
        p.set_option(H.HPCCG_OPT_PERSISTENT, 0)
        outs = []
        for defer in (0, 2, 3, 8):
            p.set_option(H.HPCCG_OPT_DEFER_X, defer)
            for mode in ("while", "graph", "timing"):
                p.set_option(H.HPCCG_OPT_WHILE, 1 if mode == "while" else 0)
                p.set_option(H.HPCCG_OPT_TIMING, 1 if mode == "timing" else 0)
                p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n))
                r = p.solve(max_iter, tol)
                assert p.stats()["x_deferred"] == (defer if defer >= 2 else 0), (defer, mode)
                outs.append((r["niters"], r["normr"], p.get_vec(H.HPCCG_VEC_X)))
        for k, v in ((H.HPCCG_OPT_TIMING, 0), (H.HPCCG_OPT_WHILE, 1), (H.HPCCG_OPT_DEFER_X, -1),
                     (H.HPCCG_OPT_CG_VARIANT, 0)):
            p.set_option(k, v)
        for o in outs[1:]:
            assert o[:2] == outs[0][:2]
            np.testing.assert_array_equal(o[2], outs[0][2])


@pytest.mark.parametrize("P,dims", [(2, (16, 12, 6)), (3, (10, 6, 1))])
def test_sr_ring_fused_loopback_bitwise(P, dims):
    """The same on loopback z-slabs with f2's exchange fused into its kernels
    (HALO_PEER 2; the flush pass pushes r's boundary planes with its own
    pushing-block count; nz = 1: every row is a boundary row)."""
    with H.Context(0, nranks=P, loopback=True) as c, H.Problem(c, *dims) as p:
        sr(p)
        p.set_option(H.HPCCG_OPT_HALO_PEER, 2)
        outs = []
        for defer in (0, 3, 8):
            p.set_option(H.HPCCG_OPT_DEFER_X, defer)
            p.set_vec(H.HPCCG_VEC_X, np.zeros(P * p.n))
            r = p.solve(40, 0.0)
            assert p.stats()["x_deferred"] == (defer if defer >= 2 else 0)
            outs.append((r["niters"], r["normr"], p.get_vec(H.HPCCG_VEC_X)))
        for o in outs[1:]:
            assert o[:2] == outs[0][:2]
            np.testing.assert_array_equal(o[2], outs[0][2])

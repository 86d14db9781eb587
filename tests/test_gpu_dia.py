"""GPU parity of the DIA-27 reading of the SpMV (HPCCG_OPT_SPMV_FORMAT = 1):
the 2-rows/thread kernel forms each slot's column from its stencil offset
instead of loading col[] (include/hpccg.h).  Bars: the same as the ELL
kernel -- bitwise equal to the oracle's SpMV (canonical ascending-column FMA
chain, A8) -- and, since the SpMV bits are identical, a CG solve
whose niters, normr and x are bit-for-bit those of the ELL solve (which
test_gpu_parity.py holds to the oracle)."""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H  # noqa: E402


@pytest.fixture(scope="module")
def ctx():
    c = H.Context(0)
    yield c
    c.close()


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float64)).cuda()


def halo_vector(xg, n, plane, rank, nranks, fill=0.0):
    xl = np.full(n + 2 * plane, fill)
    lo = rank * n - plane
    for j in range(n + 2 * plane):
        g = lo + j
        if plane <= j < plane + n and 0 <= g < xg.size:
            xl[j] = xg[g]
    return xl


# (2, 1, 1) / (7, 5, 6): odd n or plane -> 1-row kernel (ELL) under format 1
@pytest.mark.parametrize("dims", [(20, 30, 10), (64, 64, 16), (33, 10, 3), (2, 2, 1), (8, 2, 5),
                                  (7, 5, 6), (2, 1, 1), (130, 2, 3)])
def test_dia_spmv_bitwise_vs_oracle(ctx, dims):
    nx, ny, nz = dims
    with H.Problem(ctx, nx, ny, nz) as p:
        p.set_option(H.HPCCG_OPT_SPMV_FORMAT, 1)
        ref = oracle.generate(nx, ny, nz)
        for seed in (21, 22):
            x = synth.uniform(ref.n, seed)
            y = torch.empty(ref.n, dtype=torch.float64, device="cuda")
            p.spmv(dev(halo_vector(x, ref.n, nx * ny, 0, 1, fill=np.nan)), y)
            np.testing.assert_array_equal(y.cpu().numpy(), oracle.spmv(ref, x))
        y = torch.empty(ref.n, dtype=torch.float64, device="cuda")
        p.spmv(dev(halo_vector(np.ones(ref.n), ref.n, nx * ny, 0, 1)), y)
        np.testing.assert_array_equal(y.cpu().numpy(), ref.b)      # A.1 = b


@pytest.mark.parametrize("P", [2, 3])
def test_dia_spmv_loopback_halos(P):
    """z-slabs: the DIA columns of the boundary planes reach into the halo
    planes exactly as the ELL columns do (NaN-poisoned halos refilled by the
    exchange); global oracle rows, bitwise."""
    nx, ny, nz = 10, 6, 4
    with H.Context(0, nranks=P, loopback=True) as c, H.Problem(c, nx, ny, nz) as p:
        p.set_option(H.HPCCG_OPT_SPMV_FORMAT, 1)
        g = oracle.generate(nx, ny, nz * P)
        xg = synth.uniform(g.n, 33)
        n, plane = p.n, nx * ny
        xs = np.concatenate([halo_vector(xg, n, plane, r, P, fill=np.nan) for r in range(P)])
        y = torch.empty(P * n, dtype=torch.float64, device="cuda")
        p.spmv(dev(xs), y)
        np.testing.assert_array_equal(y.cpu().numpy(), oracle.spmv(g, xg))


def _solve(p, fmt, max_iter, tol, while_graph=1, variant=0):
    p.set_option(H.HPCCG_OPT_SPMV_FORMAT, fmt)
    p.set_option(H.HPCCG_OPT_WHILE, while_graph)
    p.set_option(H.HPCCG_OPT_CG_VARIANT, variant)
    p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n * p.ctx.nslabs))
    r = p.solve(max_iter, tol)
    return r["niters"], r["normr"], p.get_vec(H.HPCCG_VEC_X)


@pytest.mark.parametrize("dims,max_iter,tol", [((24, 20, 12), 150, 1e-12), ((64, 64, 32), 41, 0.0),
                                               ((40, 30, 21), 150, 1e-12)])
@pytest.mark.parametrize("variant", [0, 1])
def test_dia_cg_bitwise_equal_to_ell(ctx, dims, max_iter, tol, variant):
    with H.Problem(ctx, *dims) as p:
        p.set_option(H.HPCCG_OPT_PERSISTENT, 0)
        outs = [_solve(p, fmt, max_iter, tol, wh, variant) for fmt in (0, 1) for wh in (1, 0)]
    for o in outs[1:]:
        assert o[:2] == outs[0][:2]
        np.testing.assert_array_equal(o[2], outs[0][2])


def test_dia_cg_vs_oracle_and_loopback(ctx):
    """Against the oracle directly (niters +-1, 1e-10), single slab and P = 2
    loopback slabs; and the option's range check."""
    nx, ny, nz = 16, 12, 6
    ref = oracle.generate(nx, ny, 2 * nz)
    oref = oracle.cg(ref, 150, 1e-12)
    with H.Problem(ctx, nx, ny, 2 * nz) as p:
        p.set_option(H.HPCCG_OPT_PERSISTENT, 0)
        it, nr, x = _solve(p, 1, 150, 1e-12)
        assert abs(it - oref["niters"]) <= 1
        assert abs(nr - oref["normr"]) <= 1e-10
        assert np.max(np.abs(x - oref["x"])) <= 1e-10
        with pytest.raises(H.HpccgError):
            p.set_option(H.HPCCG_OPT_SPMV_FORMAT, 2)
    with H.Context(0, nranks=2, loopback=True) as c, H.Problem(c, nx, ny, nz) as p:
        it, nr, x = _solve(p, 1, 150, 1e-12)
        assert abs(it - oref["niters"]) <= 1
        assert abs(nr - oref["normr"]) <= 1e-10
        assert np.max(np.abs(x - oref["x"])) <= 1e-10


def test_dia_full_128cubed_bitwise_to_ell(ctx):
    """The bench's hpccg128 launch configuration (while-graph, 2 rows/thread):
    500 iterations (tol 0) give the ELL run's bits."""
    with H.Problem(ctx, 128, 128, 128) as p:
        a = _solve(p, 0, 500, 0.0)
        b = _solve(p, 1, 500, 0.0)
    assert a[:2] == b[:2]
    np.testing.assert_array_equal(a[2], b[2])


@pytest.mark.parametrize("P,dims", [(2, (12, 10, 6)), (3, (8, 8, 2)), (2, (16, 16, 1))])
def test_dia_fused_peer_path_bitwise(P, dims):
    """HALO_PEER = 2 (halo push / wait and allreduces fused into the CG
    kernels): the DIA reading of the boundary blocks' halo gathers (coherent
    loads after the flag wait) gives the ELL run's bits, for both CG variants
    and every exchange mode."""
    nx, ny, nz = dims
    with H.Context(0, nranks=P, loopback=True) as c, H.Problem(c, nx, ny, nz) as p:
        for variant in (0, 1):
            outs = []
            for fmt, peer in [(0, 2), (1, 2), (1, 1), (1, 0)]:
                p.set_option(H.HPCCG_OPT_HALO_PEER, peer)
                p.set_option(H.HPCCG_OPT_SPMV_FORMAT, fmt)
                p.set_option(H.HPCCG_OPT_CG_VARIANT, variant)
                p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n * P))
                r = p.solve(150, 1e-12)
                outs.append((r["niters"], r["normr"], p.get_vec(H.HPCCG_VEC_X)))
            for o in outs[1:]:
                assert o[:2] == outs[0][:2]
                np.testing.assert_array_equal(o[2], outs[0][2])


@pytest.mark.parametrize("variant", [0, 1])
def test_dia_on_chip_solve(ctx, variant):
    """The shared-memory-resident cluster solve under format 1 drops the
    column slice where the ELL slice does not fit (216 + 40/48 B per row
    instead of 324 + 40/48): same bits as ELL where both run on chip
    (20x30x10, which keeps the column slice), and it takes problems the ELL
    slice does not fit (30x20x20 = 12000 rows: ELL -> while-graph, DIA -> on
    chip), which match the oracle."""
    with H.Problem(ctx, 20, 30, 10) as p:
        outs = []
        for fmt in (0, 1):
            outs.append(_solve(p, fmt, 150, 1e-12, variant=variant))
            assert p.stats()["graph_mode"] == 5
        assert outs[1][:2] == outs[0][:2]
        np.testing.assert_array_equal(outs[1][2], outs[0][2])
    dims = (30, 20, 20)
    ref = oracle.generate(*dims)
    oref = (oracle.cg_sr if variant else oracle.cg)(ref, 150, 1e-12)
    with H.Problem(ctx, *dims) as p:
        modes = []
        for fmt in (0, 1):
            it, nr, x = _solve(p, fmt, 150, 1e-12, variant=variant)
            modes.append(p.stats()["graph_mode"])
            assert abs(it - oref["niters"]) <= 1
            assert abs(nr - oref["normr"]) <= 1e-10
            assert np.max(np.abs(x - oref["x"])) <= 1e-10
        assert modes == [2, 5]

"""Two z-slab ranks as two PROCESSES on one GPU, peer-only contexts: the
multi-process HALO_PEER path (CUDA IPC export / open, neighbour halo pushes
and allreduce posts into another process's memory, release/acquire flags)
against the global oracle and bit-for-bit against the same decomposition in
one process (loopback + HALO_PEER, whose reduction order it shares)."""
import multiprocessing as mp

import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H  # noqa: E402


def run_ranks(nranks, dims, variant, max_iter, tol, timeout=240, halo=1, defer=None,  # noqa: PLR0913
              defer_after=None):
    import peer_worker
    ctx = mp.get_context("spawn")
    to_parent = ctx.Queue()
    inbox = [ctx.Queue() for _ in range(nranks)]
    procs = [ctx.Process(target=peer_worker.run,
                         args=(r, nranks, dims, variant, max_iter, tol, to_parent, inbox[r], halo, defer,
                               defer_after))
             for r in range(nranks)]
    for pr in procs:
        pr.start()
    try:
        blobs, done = {}, {}
        while len(blobs) < nranks:
            kind, r, payload = to_parent.get(timeout=timeout)
            assert kind == "blob", payload
            blobs[r] = payload
        for q in inbox:
            q.put([blobs[r] for r in range(nranks)])
        while len(done) < nranks:
            kind, r, payload = to_parent.get(timeout=timeout)
            assert kind == "done", payload
            done[r] = payload
        return [done[r] for r in range(nranks)]
    finally:
        for pr in procs:
            pr.join(timeout=30)
            if pr.is_alive():
                pr.kill()


@pytest.mark.parametrize("variant", [0, 1])
def test_two_processes_one_gpu_peer_cg(variant):
    P, dims = 2, (16, 12, 6)
    res = run_ranks(P, dims, variant, 150, 1e-12)
    ref = oracle.generate(dims[0], dims[1], dims[2] * P)
    oref = (oracle.cg_sr if variant else oracle.cg)(ref, 150, 1e-12)
    with H.Context(0, nranks=P, loopback=True) as c, H.Problem(c, *dims) as p:
        p.set_option(H.HPCCG_OPT_CG_VARIANT, variant)
        p.set_option(H.HPCCG_OPT_HALO_PEER, 1)
        rl = p.solve(150, 1e-12)
        xl = p.get_vec(H.HPCCG_VEC_X)
    for k in range(2):                       # while-graph, per-iteration graph
        outs = [res[r][k] for r in range(P)]
        assert outs[0]["mode"] == (2 if k == 0 else 1)
        assert outs[0]["nnz_global"] == ref.nnz
        x = np.concatenate([o["x"] for o in outs])
        for o in outs:                       # every rank took the same decisions
            assert (o["niters"], o["normr"]) == (rl["niters"], rl["normr"])
            assert o["err"] == outs[0]["err"]
        np.testing.assert_array_equal(x, xl)
        assert abs(outs[0]["niters"] - oref["niters"]) <= 1
        assert np.max(np.abs(x - oref["x"])) <= 1e-10


def test_three_processes_fixed_iterations():
    P, dims = 3, (8, 8, 4)
    res = run_ranks(P, dims, 0, 12, 0.0)
    ref = oracle.generate(8, 8, 4 * P)
    oref = oracle.cg(ref, 12, 0.0)
    x = np.concatenate([res[r][0]["x"] for r in range(P)])
    assert all(res[r][0]["niters"] == 11 for r in range(P))
    assert np.max(np.abs(x - oref["x"])) <= 1e-10


@pytest.mark.parametrize("P,dims,max_iter,tol", [(2, (16, 12, 6), 150, 1e-12), (3, (8, 8, 4), 12, 0.0),
                                                 (2, (10, 6, 1), 40, 0.0)])
def test_processes_fused_peer_kernels(P, dims, max_iter, tol):
    """HALO_PEER = 2 across processes: the p update pushes its boundary planes
    into the other process's halo and raises its flag, the SpMV's boundary
    blocks wait for it and post p.Ap, the update collects every rank's p.Ap
    and posts r.r -- bit for bit the loopback HALO_PEER = 1 run, and within
    the north_star tolerance of the global oracle (nz = 1: every row touches
    both halos)."""
    res = run_ranks(P, dims, 0, max_iter, tol, halo=2)
    ref = oracle.generate(dims[0], dims[1], dims[2] * P)
    oref = oracle.cg(ref, max_iter, tol)
    with H.Context(0, nranks=P, loopback=True) as c, H.Problem(c, *dims) as p:
        p.set_option(H.HPCCG_OPT_HALO_PEER, 1)
        rl = p.solve(max_iter, tol)
        xl = p.get_vec(H.HPCCG_VEC_X)
    for k in range(2):                       # while-graph, per-iteration graph
        outs = [res[r][k] for r in range(P)]
        x = np.concatenate([o["x"] for o in outs])
        for o in outs:
            assert (o["niters"], o["normr"]) == (rl["niters"], rl["normr"])
        np.testing.assert_array_equal(x, xl)
        assert abs(outs[0]["niters"] - oref["niters"]) <= 1
        assert np.max(np.abs(x - oref["x"])) <= 1e-10


@pytest.mark.parametrize("P,dims,max_iter,tol,m", [(2, (16, 12, 6), 150, 1e-12, 8), (3, (8, 8, 4), 12, 0.0, 3),
                                                   (2, (10, 6, 1), 40, 0.0, 5)])
def test_processes_ring_deferred_x(P, dims, max_iter, tol, m):
    """HALO_PEER = 2 across processes with x deferred over m iterations: each
    rank's p ring is exported with its IPC blob, the p update pushes p_K's
    boundary planes into slot K % (m + 1) of the neighbours' rings and the
    SpMV gathers that slot -- bit for bit the same loop with x deferred by one
    iteration (loopback), in both graph modes."""
    res = run_ranks(P, dims, 0, max_iter, tol, halo=2, defer=m)
    with H.Context(0, nranks=P, loopback=True) as c, H.Problem(c, *dims) as p:
        p.set_option(H.HPCCG_OPT_HALO_PEER, 2)
        p.set_option(H.HPCCG_OPT_DEFER_X, 1)
        rl = p.solve(max_iter, tol)
        xl = p.get_vec(H.HPCCG_VEC_X)
    for k in range(2):
        outs = [res[r][k] for r in range(P)]
        x = np.concatenate([o["x"] for o in outs])
        for o in outs:
            assert o["x_deferred"] == m
            assert (o["niters"], o["normr"]) == (rl["niters"], rl["normr"])
        np.testing.assert_array_equal(x, xl)


def test_processes_ring_requested_after_exchange_falls_back():
    """A ring depth set only after the peer exchange (the neighbours mapped no
    ring): the z-slab loop falls back to x deferred by one iteration (m = 1)
    instead of pushing into unmapped rings -- same bits as loopback m = 1."""
    P, dims = 2, (16, 12, 6)
    res = run_ranks(P, dims, 0, 40, 0.0, halo=2, defer_after=5)
    with H.Context(0, nranks=P, loopback=True) as c, H.Problem(c, *dims) as p:
        p.set_option(H.HPCCG_OPT_HALO_PEER, 2)
        p.set_option(H.HPCCG_OPT_DEFER_X, 1)
        rl = p.solve(40, 0.0)
        xl = p.get_vec(H.HPCCG_VEC_X)
    for k in range(2):
        outs = [res[r][k] for r in range(P)]
        for o in outs:
            assert o["x_deferred"] == 1
            assert (o["niters"], o["normr"]) == (rl["niters"], rl["normr"])
        np.testing.assert_array_equal(np.concatenate([o["x"] for o in outs]), xl)


def test_processes_fused_peer_single_reduction():
    """f2 with HALO_PEER = 2 across 2 processes: bit for bit the loopback
    HALO_PEER = 1 run, within the tolerance of the f2 oracle."""
    P, dims = 2, (16, 12, 6)
    res = run_ranks(P, dims, 1, 150, 1e-12, halo=2)
    ref = oracle.generate(dims[0], dims[1], dims[2] * P)
    oref = oracle.cg_sr(ref, 150, 1e-12)
    with H.Context(0, nranks=P, loopback=True) as c, H.Problem(c, *dims) as p:
        p.set_option(H.HPCCG_OPT_CG_VARIANT, 1)
        p.set_option(H.HPCCG_OPT_HALO_PEER, 1)
        rl = p.solve(150, 1e-12)
        xl = p.get_vec(H.HPCCG_VEC_X)
    for k in range(2):
        outs = [res[r][k] for r in range(P)]
        x = np.concatenate([o["x"] for o in outs])
        for o in outs:
            assert (o["niters"], o["normr"]) == (rl["niters"], rl["normr"])
        np.testing.assert_array_equal(x, xl)
        assert abs(outs[0]["niters"] - oref["niters"]) <= 1
        assert np.max(np.abs(x - oref["x"])) <= 1e-10


@pytest.mark.parametrize("halo", [1, 2])
def test_peer_wait_timeout_names_rank_and_is_sticky(halo):
    """HPCCG_OPT_PEER_TIMEOUT_MS: a rank whose neighbour never joins gives up
    after the limit with HPCCG_ECUDA naming itself, what it waited for and the
    peer (no hang); the problem then refuses further solves at once."""
    import peer_worker
    P, dims = 2, (16, 12, 6)
    mctx = mp.get_context("spawn")
    to_parent = mctx.Queue()
    inbox = [mctx.Queue() for _ in range(P)]
    procs = [mctx.Process(target=peer_worker.run_timeout, args=(r, P, dims, halo, to_parent, inbox[r]))
             for r in range(P)]
    for pr in procs:
        pr.start()
    try:
        blobs = {}
        while len(blobs) < P:
            kind, r, payload = to_parent.get(timeout=240)
            assert kind == "blob", payload
            blobs[r] = payload
        for q in inbox:
            q.put([blobs[r] for r in range(P)])
        kind, r, out = to_parent.get(timeout=240)
        assert kind == "done" and r == 0, out
        inbox[1].put("go")
        kind, r1, _ = to_parent.get(timeout=240)
        assert kind == "done" and r1 == 1
    finally:
        for pr in procs:
            pr.join(timeout=30)
            if pr.is_alive():
                pr.kill()
    st, code, msg, secs = out["first"]
    assert st == "error" and code == H.HPCCG_ECUDA, out
    assert "timed out after 300 ms on rank 0" in msg and "rank 1" in msg, msg
    assert secs < 20, secs
    st2, code2, msg2, secs2 = out["second"]
    assert st2 == "error" and code2 == H.HPCCG_ECUDA and "recreate" in msg2 and secs2 < 5, out


def test_halo_peer_value_checked_before_mapping():
    """An out-of-range HALO_PEER is refused (EINVAL) before any peer mapping or
    collective is attempted (1-rank NCCL context)."""
    uid = H.hpccg_unique_id()
    with H.Context(0, rank=0, nranks=1, unique_id=uid) as c, H.Problem(c, 8, 8, 4) as p:
        for bad in (3, -1):
            with pytest.raises(H.HpccgError) as e:
                p.set_option(H.HPCCG_OPT_HALO_PEER, bad)
            assert e.value.code == H.HPCCG_EINVAL
        with pytest.raises(H.HpccgError) as e:
            p.set_option(H.HPCCG_OPT_PEER_TIMEOUT_MS, 0)
        assert e.value.code == H.HPCCG_EINVAL
        p.set_option(H.HPCCG_OPT_PEER_TIMEOUT_MS, 45000)
        r = p.solve(50, 1e-12)
        assert r["niters"] > 0

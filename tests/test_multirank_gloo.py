"""World-size-2 ``gloo`` tests on CPU of the N > 1 path's host logic:

* the NCCL unique-id bootstrap over torch.distributed (real hpccg_unique_id),
* the z-slab decomposition helpers bench.py uses (weak / strong),
* max-over-ranks timing aggregation,
* the decomposition protocol itself: a slab-distributed HPCCG CG whose halo
  exchange (first owned plane -> rank-1's upper halo, last owned plane ->
  rank+1's lower halo) and per-dot allreduce run over gloo, built from the
  oracle's slab kernels, reproduces the single global oracle problem
  (the GPU library uses the same layout and protocol).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _run(fn, world, *args):
    port = _free_port()
    mp.spawn(_entry, args=(world, port, fn, args), nprocs=world, join=True)


def _entry(rank, world, port, fn, args):
    import sys
    sys.path.insert(0, ROOT)
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    try:
        fn(rank, world, *args)
    finally:
        dist.destroy_process_group()


# ------------------------------------------------------------------ bodies

def _body_bootstrap(rank, world):
    from paper_conf_sc_valero_laragmtv24_b200 import dist as D
    from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
    uid = D.broadcast_unique_id(H.hpccg_unique_id)
    assert len(uid) == 128
    got = [None] * world
    dist.all_gather_object(got, uid)
    assert all(g == uid for g in got)
    t, w = D.max_time_sum_work(10.0 * (rank + 1), 3.0)
    assert t == 10.0 * world and w == 3.0 * world


def _halo_exchange(xl, s):
    """The protocol of the library's exchange(), over gloo point-to-point."""
    n, pl = s.n, s.plane
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a))  # noqa: E731
    reqs = []
    lo = torch.zeros(pl, dtype=torch.float64)
    hi = torch.zeros(pl, dtype=torch.float64)
    if s.rank > 0:
        reqs.append(dist.isend(t(xl[pl:2 * pl]), s.rank - 1))
        reqs.append(dist.irecv(lo, s.rank - 1))
    if s.rank < s.nranks - 1:
        reqs.append(dist.isend(t(xl[n:n + pl]), s.rank + 1))
        reqs.append(dist.irecv(hi, s.rank + 1))
    for r in reqs:
        r.wait()
    xl[:pl] = lo.numpy()
    xl[pl + n:] = hi.numpy()


def _allsum(v):
    t = torch.tensor([v], dtype=torch.float64)
    dist.all_reduce(t)
    return float(t.item())


def _body_distributed_cg(rank, world, nx, ny, nz, max_iter, tol):
    import oracle
    from paper_conf_sc_valero_laragmtv24_b200 import dist as D
    s = D.slab_for(nx, ny, nz, rank, world, "weak")
    prob = oracle.generate(nx, ny, nz, rank, world)
    assert prob.col_offset == s.col_offset
    n, pl = s.n, s.plane
    x = np.zeros(n)
    r = np.empty(n)
    pl_vec = np.zeros(n + 2 * pl)              # p with halos

    def spmv(pv):
        _halo_exchange(pv, s)
        return oracle.spmv(prob, pv, s.col_offset)

    pl_vec[pl:pl + n] = x
    Ap = spmv(pl_vec)
    oracle.waxpby(1.0, prob.b, -1.0, Ap, out=r)
    rtrans = _allsum(oracle.ddot(r, r))
    normr = np.sqrt(rtrans)
    niters = 0
    k = 1
    while k < max_iter and normr > tol:
        p = pl_vec[pl:pl + n]
        if k == 1:
            p[:] = r
        else:
            old, rtrans = rtrans, _allsum(oracle.ddot(r, r))
            p[:] = oracle.waxpby(1.0, r, rtrans / old, p.copy())
        normr = np.sqrt(rtrans)
        Ap = spmv(pl_vec)
        pAp = _allsum(oracle.ddot(pl_vec[pl:pl + n], Ap))
        stop = rtrans == 0.0 or pAp == 0.0
        alpha = 0.0 if stop else rtrans / pAp
        oracle.waxpby(1.0, x, alpha, pl_vec[pl:pl + n].copy(), out=x)
        oracle.waxpby(1.0, r, -alpha, Ap, out=r)
        niters = k
        k += 1
        if stop:
            break
    xs = [None] * world
    dist.all_gather_object(xs, x)
    if rank == 0:
        g = oracle.generate(nx, ny, nz * world)
        ref = oracle.cg(g, max_iter, tol)
        assert abs(niters - ref["niters"]) <= 1, (niters, ref["niters"])
        assert abs(normr - ref["normr"]) <= 1e-10
        xg = np.concatenate(xs)
        assert np.max(np.abs(xg - ref["x"])) <= 1e-10
        assert oracle.maxabsdiff(xg, g.xexact) <= 1e-12


def _body_peer_blobs(rank, world):
    from paper_conf_sc_valero_laragmtv24_b200 import dist as D
    blob = bytes([rank + 1]) * 256
    got = D.allgather_peer_blobs(blob)
    assert got == [bytes([r + 1]) * 256 for r in range(world)]
    with pytest.raises(ValueError):
        D.allgather_peer_blobs(b"short")


# ------------------------------------------------------------------- tests

def test_gloo_peer_blob_allgather():
    """Peer-only contexts: the caller all-gathers the hpccg_peer_export blobs
    (rank order) before hpccg_peer_attach."""
    _run(_body_peer_blobs, 3)



def test_slab_helpers():
    from paper_conf_sc_valero_laragmtv24_b200 import dist as D
    w = D.slab_for(256, 256, 256, 3, 8, "weak")
    assert (w.nz, w.nz_global, w.row0, w.col_offset) == (256, 2048, 3 * 256 ** 3,
                                                          3 * 256 ** 3 - 256 ** 2)
    s = D.slab_for(512, 512, 512, 7, 8, "strong")
    assert s.nz == 64 and s.nz_global == 512
    with pytest.raises(ValueError):
        D.slab_for(8, 8, 10, 0, 3, "strong")


def test_gloo_bootstrap_unique_id_and_aggregation():
    _run(_body_bootstrap, 2)


@pytest.mark.parametrize("dims", [(9, 7, 4), (12, 10, 1)])
def test_gloo_zslab_cg_matches_global_oracle(dims):
    _run(_body_distributed_cg, 2, *dims, 150, 1e-12)


def _body_peer_decision(rank, world, fail_rank, fail_stage):
    """bench.py's fallback decision (dist.decide_peer_path) over gloo: one rank's
    IPC mapping (or proof solve) fails -> EVERY rank resets to NCCL and reports
    the same stage and failing rank; nobody proceeds to the proof after a map
    failure."""
    from paper_conf_sc_valero_laragmtv24_b200 import dist as D
    calls = []

    def stage_fn(stage):
        def fn():
            calls.append(stage)
            if rank == fail_rank and stage == fail_stage:
                raise RuntimeError(f"hpccg_set_option: cudaIpcOpenMemHandle failed on rank {rank}")
        return fn

    dec = D.decide_peer_path(stage_fn("map"), stage_fn("proof"), stage_fn("reset"))
    got = [None] * world
    dist.all_gather_object(got, dec)
    assert all(g == got[0] for g in got), got            # the same decision everywhere
    if fail_rank is None:
        assert dec["peer"] is True and calls == ["map", "proof"]
        return
    assert dec["peer"] is False and dec["stage"] == fail_stage
    assert dec["failed_ranks"] == [fail_rank] and str(fail_rank) in dec["errors"]
    assert f"rank {fail_rank}" in dec["why"]
    want = ["map", "reset"] if fail_stage == "map" else ["map", "proof", "reset"]
    assert calls == want, calls


@pytest.mark.parametrize("fail_rank,fail_stage", [(None, None), (1, "map"), (0, "map"), (1, "proof")])
def test_gloo_peer_path_fallback_decision(fail_rank, fail_stage):
    _run(_body_peer_decision, 2, fail_rank, fail_stage)

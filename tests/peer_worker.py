"""Child-process body of tests/test_gpu_peer_ipc.py (not a test module).

One z-slab rank in its own process on GPU 0, in a PEER-ONLY context (no
NCCL): export the CUDA-IPC blob, receive every rank's blob from the parent,
attach, solve, and report.  Ranks on one GPU exercise the real multi-process
path of HPCCG_OPT_HALO_PEER -- IPC export / open, peer tables, cross-process
flags and allreduce slots -- that NCCL cannot (it refuses two ranks on one
GPU)."""


def run(rank, nranks, dims, variant, max_iter, tol, to_parent, from_parent, halo=1, defer=None,
        defer_after=None):
    try:
        import numpy as np
        from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
        with H.Context(0, rank=rank, nranks=nranks, peer=True) as c, H.Problem(c, *dims) as p:
            p.set_option(H.HPCCG_OPT_CG_VARIANT, variant)
            if defer is not None:  # before the export: a ring is exchanged with the blob
                p.set_option(H.HPCCG_OPT_DEFER_X, defer)
            to_parent.put(("blob", rank, p.peer_export()))
            blobs = from_parent.get(timeout=120)
            p.peer_attach(blobs)
            if halo != 1:  # 2: exchange + allreduces fused into the CG kernels
                p.set_option(H.HPCCG_OPT_HALO_PEER, halo)
            if defer_after is not None:  # a ring allocated after the exchange: not addressed
                p.set_option(H.HPCCG_OPT_DEFER_X, defer_after)
            out = []
            for wh in (1, 0):
                p.set_option(H.HPCCG_OPT_WHILE, wh)
                p.set_vec(H.HPCCG_VEC_X, np.zeros(p.n))
                r = p.solve(max_iter, tol)
                out.append({"niters": r["niters"], "normr": r["normr"], "err": p.maxabsdiff(),
                            "x": p.get_vec(H.HPCCG_VEC_X), "mode": p.stats()["graph_mode"],
                            "nnz_global": p.info["nnz_global"], "x_deferred": p.stats()["x_deferred"]})
            to_parent.put(("done", rank, out))
    except Exception as e:  # reported to the parent, which fails the test
        to_parent.put(("error", rank, repr(e)))


def run_maxabs(rank, nranks, dims, x_slab, xe_slab, to_parent, from_parent):
    """a.9 across processes: set this rank's X (and X_EXACT) slab, then the
    collective max|x - x_exact| (local kernel + peer MAX allreduce)."""
    try:
        from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
        with H.Context(0, rank=rank, nranks=nranks, peer=True) as c, H.Problem(c, *dims) as p:
            to_parent.put(("blob", rank, p.peer_export()))
            p.peer_attach(from_parent.get(timeout=120))
            p.set_vec(H.HPCCG_VEC_X, x_slab)
            if xe_slab is not None:
                p.set_vec(H.HPCCG_VEC_XEXACT, xe_slab)
            to_parent.put(("done", rank, p.maxabsdiff()))
    except Exception as e:
        to_parent.put(("error", rank, repr(e)))


def run_timeout(rank, nranks, dims, halo, to_parent, from_parent):
    """Rank 0 solves with a short peer-wait limit while rank 1 never joins: the
    solve must fail with HPCCG_ECUDA naming both ranks (no hang), and a second
    solve of the same problem must refuse at once (sticky record)."""
    try:
        import time

        from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H
        with H.Context(0, rank=rank, nranks=nranks, peer=True) as c, H.Problem(c, *dims) as p:
            to_parent.put(("blob", rank, p.peer_export()))
            p.peer_attach(from_parent.get(timeout=120))
            p.set_option(H.HPCCG_OPT_HALO_PEER, halo)
            out = {}
            if rank == 0:
                p.set_option(H.HPCCG_OPT_PEER_TIMEOUT_MS, 300)
                for k in ("first", "second"):
                    t0 = time.perf_counter()
                    try:
                        p.solve(20, 0.0)
                        out[k] = ("ok", 0, "", 0.0)
                    except H.HpccgError as e:
                        out[k] = ("error", e.code, str(e), time.perf_counter() - t0)
            else:
                from_parent.get(timeout=120)      # released after rank 0 reported
            to_parent.put(("done", rank, out))
    except Exception as e:
        to_parent.put(("error", rank, repr(e)))

"""Host-side plumbing of the multi-GPU z-slab path (north_star "z-slab
decomposition across the 8 B200s").

torch.distributed is only the bootstrap: it broadcasts the 128-byte NCCL
unique id (the library then owns its NCCL communicator, halo exchange and
scalar allreduces) and aggregates the bench timings (max over ranks).
"""
from __future__ import annotations

from dataclasses import dataclass


@dataclass(frozen=True)
class Slab:
    nx: int
    ny: int
    nz: int          # local z-planes of this rank
    rank: int
    nranks: int

    @property
    def n(self) -> int:
        return self.nx * self.ny * self.nz

    @property
    def plane(self) -> int:
        return self.nx * self.ny

    @property
    def row0(self) -> int:
        """Global id of the first owned row."""
        return self.rank * self.n

    @property
    def col_offset(self) -> int:
        """Global id of local-with-halo index 0: [lower halo | owned | upper halo]."""
        return self.row0 - self.plane

    @property
    def nz_global(self) -> int:
        return self.nz * self.nranks


def slab_for(nx: int, ny: int, nz: int, rank: int, nranks: int, scaling: str) -> Slab:
    """weak: nz planes per rank (global nz * nranks); strong: the global nz is
    split evenly (A13: 512^3 -> 512 / P planes per rank)."""
    if nranks < 1 or not 0 <= rank < nranks:
        raise ValueError("bad rank / nranks")
    if scaling == "weak":
        return Slab(nx, ny, nz, rank, nranks)
    if scaling == "strong":
        if nz % nranks:
            raise ValueError(f"strong scaling needs nz ({nz}) divisible by nranks ({nranks})")
        return Slab(nx, ny, nz // nranks, rank, nranks)
    raise ValueError(scaling)


def broadcast_unique_id(make_id, src: int = 0) -> bytes:
    """Rank `src` calls make_id() (hpccg_unique_id); every rank returns it."""
    import torch.distributed as dist
    obj = [make_id() if dist.get_rank() == src else None]
    dist.broadcast_object_list(obj, src=src)
    uid = obj[0]
    if not isinstance(uid, (bytes, bytearray)) or len(uid) != 128:
        raise RuntimeError("bad NCCL unique id from rank %d" % src)
    return bytes(uid)


def allgather_peer_blobs(blob: bytes, nbytes: int = 256) -> list:
    """Every rank's hpccg_peer_export blob, in rank order (for peer-only
    contexts, which have no NCCL: hpccg_peer_attach takes the list)."""
    import torch.distributed as dist
    if len(blob) != nbytes:
        raise ValueError("peer blob must be %d bytes" % nbytes)
    got = [None] * dist.get_world_size()
    dist.all_gather_object(got, bytes(blob))
    if any(not isinstance(b, (bytes, bytearray)) or len(b) != nbytes for b in got):
        raise RuntimeError("bad peer blob from a rank")
    return [bytes(b) for b in got]


def max_time_sum_work(ms_local: float, work_local: float, device=None):
    """(max over ranks of the device time, sum over ranks of the work)."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([ms_local], dtype=torch.float64, device=device)
    w = torch.tensor([work_local], dtype=torch.float64, device=device)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.all_reduce(w, op=dist.ReduceOp.SUM)
    return float(t.item()), float(w.item())


def _attempt(fn):
    """None if fn() returns, else the exception as one line."""
    try:
        fn()
        return None
    except Exception as e:  # noqa: BLE001 -- every failure is reported, none is fatal here
        return f"{type(e).__name__}: {e}".replace("\n", " ")[:300]


def _gather_objects(obj):
    import torch.distributed as dist
    out = [None] * dist.get_world_size()
    dist.all_gather_object(out, obj)
    return out


def decide_peer_path(try_map, try_proof, reset, gather=None) -> dict:
    """Agree, on every rank, whether the multi-GPU solve runs over peer memory
    (HPCCG_OPT_HALO_PEER) or falls back to NCCL send/recv + allreduce.

    Two collective stages, each followed by an all-gather of every rank's
    outcome so all ranks take the SAME decision (a rank on the peer path and
    one on NCCL would wait on each other forever):
      1. try_map()   -- map the neighbours' buffers (CUDA IPC over NVLink);
      2. try_proof() -- a short solve that exercises the mapping end to end.
    If any rank failed a stage, every rank calls reset() (HALO_PEER = 0) and the
    result names the stage, the failing ranks and their errors."""
    gather = gather or _gather_objects
    for stage, fn in (("map", try_map), ("proof", try_proof)):
        errs = gather(_attempt(fn))
        failed = {r: e for r, e in enumerate(errs) if e}
        if failed:
            reset_err = _attempt(reset)
            first = min(failed)
            return {"peer": False, "stage": stage, "failed_ranks": sorted(failed),
                    "errors": {str(r): e for r, e in failed.items()}, "reset_error": reset_err,
                    "why": f"{stage} failed on rank(s) {sorted(failed)}: {failed[first]}"}
    return {"peer": True, "stage": "proof", "failed_ranks": [], "errors": {}, "reset_error": None,
            "why": None}

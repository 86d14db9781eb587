"""CPU model of the HALO_PEER = 2 protocol (kernels.cuh "HALO_PEER = 2"):
P ranks as threads with random delays run the fused iteration's
communication -- the slab sums posted into LL slots (slot 1: p.Ap, seq
2k - 1; slot 0: r.r, seq 2k; exact tag match), the p planes pushed into the
neighbours' halo buffers and their flags raised with tag(epoch, k) -- in the
order the three kernels issue them, across several solves (epochs).

It checks the two claims the design rests on, under arbitrary interleavings:
(1) no slot is overwritten before every rank has collected it (a reader would
    see a foreign tag and never finish: caught by the timeout) and every
    collect returns the values of its own iteration;
(2) no halo is overwritten before the neighbour's SpMV has read it: every
    halo read returns the neighbour's p of the same iteration.
The device-side memory ordering (fences, single-copy atomic 8-B words) is
not modelled: each write here is atomic."""
import random
import threading
import time

import pytest


class Shared:
    def __init__(self, P):
        self.P = P
        # slots[owner][q][writer] = (tag, value)
        self.slots = [[[(0, None)] * P for _ in range(2)] for _ in range(P)]
        self.halo = [[None, None] for _ in range(P)]     # [owner][0 lower | 1 upper] = value
        self.flag = [[0, 0] for _ in range(P)]           # [owner][0 from lo | 1 from hi]
        self.barrier = threading.Barrier(P)   # the host sync at the end of every solve
        self.errors = []


def ll_tag(epoch, seq):  # kernels.cuh ll_tag
    return 0x80000000 | ((epoch & 0x7FF) << 20) | (seq & 0xFFFFF)


def ftag(epoch, seq):    # kernels.cuh ftag
    return (epoch << 32) | seq


def spin(pred, deadline):
    while not pred():
        if time.monotonic() > deadline:
            return False
        time.sleep(0)
    return True


def rank_main(sh, r, solves, iters, seed, deadline, one_slot=False):
    rnd = random.Random(seed)
    P = sh.P

    def jitter():
        if rnd.random() < 0.5:
            time.sleep(rnd.random() * 2e-4)

    def post(q, seq, epoch, value):
        for dst in range(P):
            jitter()
            sh.slots[dst][q][r] = (ll_tag(epoch, seq), value)

    def collect(q, seq, epoch, expect):
        tag = ll_tag(epoch, seq)
        got = []
        for src in range(P):
            if not spin(lambda: sh.slots[r][q][src][0] == tag, deadline):
                sh.errors.append(f"rank {r}: slot {q} seq {seq} from {src} never arrived (overwritten?)")
                return False
            got.append(sh.slots[r][q][src][1])
        if got != [expect(src) for src in range(P)]:
            sh.errors.append(f"rank {r}: slot {q} seq {seq} values {got}")
            return False
        return True

    for epoch in range(1, solves + 1):
        # init (counted exchange + allreduce of their own words): modelled as a
        # barrier-like step -- every rank finished the previous solve
        for k in range(1, iters + 1):
            # p update k: collect r.r(k-1), then push p(k) into the neighbours' halos
            if k > 1:
                post(0, 2 * (k - 1), epoch, ("rr", epoch, k - 1, r))
                if not collect(0, 2 * (k - 1), epoch, lambda s: ("rr", epoch, k - 1, s)):
                    return
            for nb, side in ((r - 1, 1), (r + 1, 0)):   # my first plane -> (r-1)'s upper halo
                if 0 <= nb < P:
                    jitter()
                    sh.halo[nb][side] = ("p", epoch, k, r)
            jitter()
            for nb, side in ((r - 1, 1), (r + 1, 0)):
                if 0 <= nb < P:
                    sh.flag[nb][side] = ftag(epoch, k)
            # SpMV k: the boundary blocks wait for the flags, then read the halos
            for nb, side in ((r - 1, 0), (r + 1, 1)):
                if 0 <= nb < P:
                    if not spin(lambda: sh.flag[r][side] >= ftag(epoch, k), deadline):
                        sh.errors.append(f"rank {r}: halo flag {side} of iteration {k} never raised")
                        return
                    jitter()
                    v = sh.halo[r][side]
                    if v != ("p", epoch, k, nb):
                        sh.errors.append(f"rank {r}: halo {side} at iteration {k} read {v}")
                        return
            # update k: post p.Ap(k), collect it
            q1 = 0 if one_slot else 1
            post(q1, 2 * k - 1, epoch, ("pAp", epoch, k, r))
            if not collect(q1, 2 * k - 1, epoch, lambda s: ("pAp", epoch, k, s)):
                return
        # the solve ends with the host synchronising every rank (maxabsdiff allreduce)
        sh_barrier(sh, P)


def sh_barrier(sh, P):
    try:
        sh.barrier.wait(timeout=20)
    except threading.BrokenBarrierError:
        sh.errors.append("solve-end barrier broken (a rank stopped early)")


@pytest.mark.parametrize("P", [1, 2, 3, 5, 8])
def test_fused_protocol_interleavings(P):
    sh = Shared(P)
    deadline = time.monotonic() + 60
    th = [threading.Thread(target=rank_main, args=(sh, r, 3, 12, 1000 * P + r, deadline))
          for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=90)
    assert not any(t.is_alive() for t in th), "deadlock"
    assert not sh.errors, sh.errors[:3]


def test_model_detects_a_broken_protocol():
    """Sanity of the model itself: with ONE slot for both scalars (no seq
    parity) a fast rank overwrites a post its neighbour has not collected yet
    -- the same checks must catch it (a foreign tag: the reader times out)."""
    failures = 0
    for trial in range(6):
        sh = Shared(2)
        deadline = time.monotonic() + 2
        th = [threading.Thread(target=rank_main, args=(sh, r, 1, 40, 77 * trial + r, deadline, True))
              for r in range(2)]
        for t in th:
            t.start()
        for t in th:
            t.join(timeout=30)
        failures += bool(sh.errors)
        if failures:
            break
    assert failures, "the model never caught the single-slot protocol"

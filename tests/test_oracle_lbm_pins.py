"""Pins for the oracle of the paper's LBM workload: Fig. 10's
D2Q9 pull step and Eq. (1).

Pinned against lattice closed forms (weights sum to 1, zero first moment,
isotropic second moment), the equilibrium's moments (density, momentum and
momentum flux p (u u^T + I/3) -- these fix the 1, 3, 4.5, 1.5 coefficients),
exact streaming (a copy, so bitwise shifts), per-site conservation of mass and
momentum by the collision, the equilibrium fixed point, and an independent
numpy transcription."""
import numpy as np
import pytest

import oracle
import synth


def test_lattice_closed_forms():
    cx, cy, w = oracle.lbm_lattice()
    assert abs(w.sum() - 1.0) < 1e-15
    assert abs((w * cx).sum()) < 1e-16 and abs((w * cy).sum()) < 1e-16
    assert abs((w * cx * cx).sum() - 1 / 3) < 1e-15 and abs((w * cy * cy).sum() - 1 / 3) < 1e-15
    assert abs((w * cx * cy).sum()) < 1e-16
    vel = set(zip(cx.tolist(), cy.tolist()))
    assert vel == {(a, b) for a in (-1, 0, 1) for b in (-1, 0, 1)}


@pytest.mark.parametrize("p,u,v", [(1.0, 0.0, 0.0), (1.3, 0.05, -0.02), (0.7, -0.1, 0.08)])
def test_feq_moments(p, u, v):
    cx, cy, _ = oracle.lbm_lattice()
    fe = np.array([oracle.lbm_feq(k, p, u, v) for k in range(9)])
    assert abs(fe.sum() - p) < 1e-14
    assert abs((fe * cx).sum() - p * u) < 1e-14 and abs((fe * cy).sum() - p * v) < 1e-14
    assert abs((fe * cx * cx).sum() - p * (u * u + 1 / 3)) < 1e-14
    assert abs((fe * cy * cy).sum() - p * (v * v + 1 / 3)) < 1e-14
    assert abs((fe * cx * cy).sum() - p * u * v) < 1e-14


def test_streaming_is_an_exact_shift():
    S = 12
    cx, cy, _ = oracle.lbm_lattice()
    f1 = synth.lbm_state(S, 3)
    f = np.full(9 * S * S, -1.0)
    f2 = np.full(9 * S * S, -2.0)
    oracle.lbm_step(S, f1, f, f2, 0.8)
    F1, F = f1.reshape(9, S, S), f.reshape(9, S, S)
    for k in range(9):
        for x in range(1, S - 1):
            for y in range(1, S - 1):
                assert F[k, x, y] == F1[k, x - int(cx[k]), y - int(cy[k])]
    # boundary sites untouched
    assert np.all(F[:, 0, :] == -1.0) and np.all(f2.reshape(9, S, S)[:, :, -1] == -2.0)


def test_collision_conserves_mass_and_momentum():
    S = 16
    cx, cy, _ = oracle.lbm_lattice()
    f1 = synth.lbm_state(S, 5, amp=0.2)
    f, f2 = np.zeros_like(f1), np.zeros_like(f1)
    oracle.lbm_step(S, f1, f, f2, 0.7)
    F, F2 = f.reshape(9, S, S)[:, 1:-1, 1:-1], f2.reshape(9, S, S)[:, 1:-1, 1:-1]
    np.testing.assert_allclose(F2.sum(0), F.sum(0), rtol=1e-14)
    np.testing.assert_allclose((F2 * cx[:, None, None]).sum(0), (F * cx[:, None, None]).sum(0),
                               atol=1e-14)
    np.testing.assert_allclose((F2 * cy[:, None, None]).sum(0), (F * cy[:, None, None]).sum(0),
                               atol=1e-14)


def test_equilibrium_is_a_fixed_point():
    S = 10
    p, u, v = 1.1, 0.04, -0.03
    fe = np.array([oracle.lbm_feq(k, p, u, v) for k in range(9)])
    f1 = np.repeat(fe, S * S).copy()
    f, f2 = np.zeros_like(f1), f1.copy()
    oracle.lbm_step(S, f1, f, f2, 0.6)
    np.testing.assert_allclose(f2, f1, rtol=1e-14)


def test_matches_independent_numpy_transcription():
    S, t = 20, 0.9
    cx, cy, w = oracle.lbm_lattice()
    f1 = synth.lbm_state(S, 7, amp=0.1)
    f, f2 = np.zeros_like(f1), np.zeros_like(f1)
    oracle.lbm_step(S, f1, f, f2, t)
    F1 = f1.reshape(9, S, S)
    Fs = np.stack([np.roll(np.roll(F1[k], int(cx[k]), 0), int(cy[k]), 1) for k in range(9)])
    Fs = Fs[:, 1:-1, 1:-1]
    p = Fs.sum(0)
    u = (Fs * cx[:, None, None]).sum(0) / p
    v = (Fs * cy[:, None, None]).sum(0) / p
    cu = cx[:, None, None] * u + cy[:, None, None] * v
    feq = w[:, None, None] * p * (1 + 3 * cu + 4.5 * cu * cu - 1.5 * (u * u + v * v))
    ref = Fs * (1 - 1 / t) + feq / t
    np.testing.assert_allclose(f2.reshape(9, S, S)[:, 1:-1, 1:-1], ref, rtol=1e-14, atol=1e-16)

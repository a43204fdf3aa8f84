"""Pins for the oracle's f1 outputs: the NAS step-0
auxiliary fields (oracle.compute_aux) and the rhs_norm numerator
(oracle.rhs_sumsq).  None retypes the oracle's formulas; each checks them
against a different characterisation:

A1  index map: u1 = 2, u2 = i, u3 = j, u4 = k (exact dyadic values) gives
    us = i/2, vs = j/2, ws = k/2, rho_i = 1/2 exactly -- catches a transposed
    axis or a wrong component.
A2  inverse relations on random fields: rho_i*u1 = 1, us*u1 = u2, vs*u1 = u3,
    ws*u1 = u4 (to rounding).
A3  square and qs from the velocities: square = (u1/2)(us^2+vs^2+ws^2) and
    qs = (us^2+vs^2+ws^2)/2 (a different evaluation of the same quantity).
A4  SP speed: speed^2 = c1c2 * (u5/u1 - (us^2+vs^2+ws^2)/2), i.e. c1c2 times
    the specific internal energy (c1c2 = 1.4*0.4 = 0.56 from the NAS gas
    constants); constant field closed form.
N1  sums of squares: a field equal to m+1 inside and 1e9 on the faces sums to
    (m+1)^2 (nx-2)(ny-2)(nz-2) exactly (faces excluded, components kept apart).
N2  NPB rms of the exact-solution residual is ~0; of a known constant interior
    it equals that constant.
"""
import numpy as np

import nasgen
import oracle


def _idx_field(nx, ny, nz):
    k, j, i = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    u = np.empty((nz, ny, nx, 5))
    u[..., 0] = 2.0
    u[..., 1] = i
    u[..., 2] = j
    u[..., 3] = k
    u[..., 4] = 50.0
    return u, i, j, k


def test_a1_index_map_exact():
    nx, ny, nz = 7, 9, 11
    u, i, j, k = _idx_field(nx, ny, nz)
    a = oracle.compute_aux(u, 7, dt=0.01)
    assert a.shape == (nz, ny, nx, 7)
    assert np.array_equal(a[..., 0], np.full((nz, ny, nx), 0.5))
    assert np.array_equal(a[..., 1], i / 2.0)
    assert np.array_equal(a[..., 2], j / 2.0)
    assert np.array_equal(a[..., 3], k / 2.0)


def test_a2_a3_relations_random_fields():
    inp = nasgen.make_inputs(9, 8, 7, seed=3, A=1e-2, dt=0.01)
    u = inp.u
    a = oracle.compute_aux(u, 6, dt=inp.dt)
    rho, us, vs, ws, sq, qs = (a[..., n] for n in range(6))
    u1 = u[..., 0]
    np.testing.assert_allclose(rho * u1, 1.0, rtol=4e-16, atol=0)
    for n, v in ((1, us), (2, vs), (3, ws)):
        np.testing.assert_allclose(v * u1, u[..., n], rtol=1e-15, atol=0)
    vel2 = us * us + vs * vs + ws * ws
    np.testing.assert_allclose(sq, 0.5 * u1 * vel2, rtol=1e-14)
    np.testing.assert_allclose(qs, 0.5 * vel2, rtol=1e-14)


def test_a4_speed_internal_energy():
    inp = nasgen.make_class("SP", "S", seed=2)
    u = inp.u
    a = oracle.compute_aux(u, 7, dt=inp.dt)
    us, vs, ws, speed = a[..., 1], a[..., 2], a[..., 3], a[..., 6]
    e_int = u[..., 4] / u[..., 0] - 0.5 * (us * us + vs * vs + ws * ws)
    np.testing.assert_allclose(speed * speed, 0.56 * e_int, rtol=1e-13)
    # constant field: speed = sqrt(0.56 * (u5 - |m|^2/(2 u1)) / u1)
    c = np.array([2.0, 1.0, -0.5, 0.25, 9.0])
    uc = np.broadcast_to(c, (6, 6, 6, 5)).copy()
    sc = oracle.compute_aux(uc, 7, dt=0.01)[..., 6]
    expect = np.sqrt(0.56 * (9.0 - (1.0 + 0.25 + 0.0625) / 4.0) / 2.0)
    np.testing.assert_allclose(sc, expect, rtol=2e-16)


def test_a_naux_validation():
    import pytest
    u = np.ones((6, 6, 6, 5))
    with pytest.raises(ValueError):
        oracle.compute_aux(u, 5, dt=0.01)


def test_n1_sumsq_interior_only_exact():
    nx, ny, nz = 8, 7, 9
    r = np.full((nz, ny, nx, 5), 1e9)
    for m in range(5):
        r[1:-1, 1:-1, 1:-1, m] = m + 1.0
    s = oracle.rhs_sumsq(r)
    n_int = (nx - 2) * (ny - 2) * (nz - 2)
    assert np.array_equal(s, np.array([(m + 1.0) ** 2 * n_int for m in range(5)]))


def test_n2_exact_solution_norm_small():
    for bench, cls in (("BT", "S"), ("SP", "W")):
        inp = nasgen.make_class(bench, cls, seed=1, A=0.0)
        r = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt)
        n = inp.nx - 2
        rms = np.sqrt(oracle.rhs_sumsq(r) / n ** 3)
        assert (rms < 1e-13 * inp.dt * 100).all(), rms

"""P7: the oracle's inviscid part against the compressible Euler equations.

This pins the NAS constants c1, c2 and tx2/ty2/tz2 (reading c2) to
textbook gas dynamics instead of to a recalled NPB constant table.  NPB BT/SP
discretise the 3-D compressible Navier-Stokes equations for an ideal gas with
gamma = 1.4 (the NPB benchmark the paper evaluates); with the
viscous (xxcon*, yycon*, zzcon*), second-order (d?tx1 ...) and fourth-order
(dssp) terms switched off, App. A steps 2, 4 and 6 must be the centred
(second-order) difference of the Euler flux vectors:

    F_x = (rho u, rho u^2 + p, rho u v, rho u w, (E + p) u),    p = (gamma - 1)(E - rho |v|^2 / 2)

so  rhs / dt  ->  -(dF_x/dx + dF_y/dy + dF_z/dz)  with error O(h^2), h = 1/(n-1).

The fluxes here are written from the primitive fields (rho, u, v, w, p), not
from the NAS expressions (c1*u5 - c2*square)*us etc., and differentiated with a
6th-order centred difference of the analytic functions, so a wrong c1, c2, a
wrong tx2 scale, a transposed velocity or a dropped pressure term shows up as a
non-converging error.  The mutant checks at the bottom prove that.
"""
import functools

import numpy as np
import pytest

import oracle

GAMMA = 1.4


def primitives(x, y, z):
    """Smooth, non-separable, positive density and pressure."""
    rho = 1.0 + 0.2 * np.sin(np.pi * x) * np.cos(0.7 * np.pi * y) + 0.1 * z
    u = 0.3 * np.sin(np.pi * y + 0.5) + 0.2 * np.cos(np.pi * z) * x + 0.25 * np.sin(1.5 * np.pi * x)
    v = -0.25 * np.cos(np.pi * x + 0.3 * z) + 0.1 * y
    w = 0.2 * np.sin(np.pi * (x + y)) - 0.15 * z * z
    p = 1.0 + 0.3 * np.cos(np.pi * x * y) + 0.2 * np.sin(np.pi * z + 0.2)
    return rho, u, v, w, p


def conservative(x, y, z):
    rho, u, v, w, p = primitives(x, y, z)
    e = p / (GAMMA - 1.0) + 0.5 * rho * (u * u + v * v + w * w)
    return np.stack([rho, rho * u, rho * v, rho * w, e], axis=-1)


def euler_flux(axis, x, y, z):
    rho, u, v, w, p = primitives(x, y, z)
    e = p / (GAMMA - 1.0) + 0.5 * rho * (u * u + v * v + w * w)
    vel = (u, v, w)[axis]
    f = [rho * vel, rho * u * vel, rho * v * vel, rho * w * vel, (e + p) * vel]
    f[1 + axis] = f[1 + axis] + p
    return np.stack(f, axis=-1)


def flux_divergence(x, y, z, h=1e-3):
    """-(div F) with a 6th-order centred difference of the analytic fluxes."""
    w6 = ((1, 45.0), (2, -9.0), (3, 1.0))
    out = 0.0
    for axis in range(3):
        d = 0.0
        for s, c in w6:
            off = [0.0, 0.0, 0.0]
            off[axis] = s * h
            plus = euler_flux(axis, x + off[0], y + off[1], z + off[2])
            minus = euler_flux(axis, x - off[0], y - off[1], z - off[2])
            d = d + c * (plus - minus)
        out = out + d / (60.0 * h)
    return -out


def inviscid_consts(n, **override):
    c = oracle.set_constants(n, n, n, 1.0)
    for name in oracle._FIELDS:
        if name.startswith(("xxcon", "yycon", "zzcon")) or name[:2] in ("dx", "dy", "dz") \
                and name.endswith(("tx1", "ty1", "tz1")):
            setattr(c, name, 0.0)
    c.dssp = 0.0
    for k, v in override.items():
        setattr(c, k, v)
    return c


def euler_error(n, **override):
    """max |rhs - (-div F)| over the interior points that lie on the 13^3 grid."""
    g = np.linspace(0.0, 1.0, n)
    z, y, x = np.meshgrid(g, g, g, indexing="ij")
    u = conservative(x, y, z)
    rhs = oracle.compute_rhs(u, np.zeros_like(u), consts=inviscid_consts(n, **override))
    want = flux_divergence(x, y, z)
    s = (n - 1) // 12
    sl = slice(s, n - s, s)  # the common interior points of the 13 / 25 / 49 grids
    err = np.abs(rhs[sl, sl, sl] - want[sl, sl, sl])
    return err.max(), np.abs(want).max()


def test_p7_inviscid_part_converges_to_euler_divergence():
    e13, scale = euler_error(13)
    e25, _ = euler_error(25)
    e49, _ = euler_error(49)
    # second-order consistency: halving h divides the error by ~4
    assert 3.5 < e13 / e25 < 4.5, (e13, e25)
    assert 3.7 < e25 / e49 < 4.3, (e25, e49)
    assert e49 < 2e-3 * scale, (e49, scale)


def test_p7_faces_are_forcing_only():
    n = 13
    g = np.linspace(0.0, 1.0, n)
    z, y, x = np.meshgrid(g, g, g, indexing="ij")
    u = conservative(x, y, z)
    rhs = oracle.compute_rhs(u, np.zeros_like(u), consts=inviscid_consts(n))
    for face in (rhs[0], rhs[-1], rhs[:, 0], rhs[:, -1], rhs[:, :, 0], rhs[:, :, -1]):
        assert np.all(face == 0.0)


@pytest.mark.parametrize("mutant", [
    {"c2": lambda c: 0.5},               # wrong gamma - 1 in the pressure
    {"c1": lambda c: 1.5},               # wrong gamma in the energy flux
    {"c1": lambda c: c.c2, "c2": lambda c: c.c1},   # c1 <-> c2 swapped
    {"tx2": lambda c: 2.0 * c.tx2},      # 1/h instead of 1/(2h) along x
    {"tz2": lambda c: c.tx2 * 0.5},      # wrong z scale
], ids=["c2", "c1", "c1c2_swap", "tx2_scale", "tz2_scale"])
def test_p7_mutated_constants_do_not_converge(mutant):
    """The pin discriminates: each mutant's error does not shrink with h."""
    def run(n):
        c = oracle.set_constants(n, n, n, 1.0)
        return euler_error(n, **{k: f(c) for k, f in mutant.items()})
    e49, _ = run(49)
    ok49, _ = euler_error(49)
    assert e49 > 5.0 * ok49, (mutant, e49, ok49)


# ----------------------------------------------------------------------------
# The full operator: Euler + NPB's Navier-Stokes viscous terms + NPB's
# second-order artificial dissipation; the fourth-order dissipation is O(h^4)
# away from the two rows next to each face.
# ----------------------------------------------------------------------------
MU = 0.1        # c3*c4: 1/Re of the NPB problem
INV_PR = 1.4    # c5: gamma / (gamma * Pr)  (NPB's 1/Pr)
ART = {0: 0.75, 1: 0.75, 2: 1.0}   # NPB dx*, dy*, dz* (all five components alike)


def d2(fn, axis, x, y, z, h=1e-2):
    """6th-order centred second derivative of an analytic field along axis."""
    wts = ((0, -490.0), (1, 270.0), (2, -27.0), (3, 2.0))
    acc = 0.0
    for s, c in wts:
        if s == 0:
            acc = acc + c * fn(x, y, z)
            continue
        off = [0.0, 0.0, 0.0]
        off[axis] = s * h
        acc = acc + c * (fn(x + off[0], y + off[1], z + off[2]) +
                         fn(x - off[0], y - off[1], z - off[2]))
    return acc / (180.0 * h * h)


def navier_stokes_viscous(x, y, z):
    """Constant-mu NS viscous terms without the cross-derivative terms (the NPB
    BT/SP model): momentum mu*(4/3 d2 u_a/da^2 + sum_{b!=a} d2 u_a/db^2);
    energy sum_a d/da[mu*((4/3) u_a du_a/da + sum_{b!=a} u_b du_b/da) + gamma*mu/Pr de/da],
    written as second derivatives of u_a^2/2 and of the internal energy e."""
    def comp(f):
        return lambda x, y, z: f(*primitives(x, y, z))
    vel = [comp(lambda r, u, v, w, p: u), comp(lambda r, u, v, w, p: v),
           comp(lambda r, u, v, w, p: w)]
    half_sq = [comp(lambda r, u, v, w, p: 0.5 * u * u), comp(lambda r, u, v, w, p: 0.5 * v * v),
               comp(lambda r, u, v, w, p: 0.5 * w * w)]
    e_int = comp(lambda r, u, v, w, p: p / ((GAMMA - 1.0) * r))
    out = []
    for m in range(3):
        out.append(MU * sum((4.0 / 3.0 if a == m else 1.0) * d2(vel[m], a, x, y, z)
                            for a in range(3)))
    en = 0.0
    for a in range(3):
        for b in range(3):
            en = en + MU * (4.0 / 3.0 if a == b else 1.0) * d2(half_sq[b], a, x, y, z)
        en = en + GAMMA * MU * INV_PR * d2(e_int, a, x, y, z)
    return np.stack([np.zeros_like(x)] + out + [en], axis=-1)


def artificial_second_order(x, y, z):
    out = 0.0
    for a in range(3):
        out = out + ART[a] * d2(conservative, a, x, y, z)
    return out


@functools.lru_cache(maxsize=None)
def _full_case(n):
    g = np.linspace(0.0, 1.0, n)
    z, y, x = np.meshgrid(g, g, g, indexing="ij")
    want = flux_divergence(x, y, z) + navier_stokes_viscous(x, y, z) + \
        artificial_second_order(x, y, z)
    return conservative(x, y, z), want


def full_error(n, consts=None):
    u, want = _full_case(n)
    c = oracle.set_constants(n, n, n, 1.0) if consts is None else consts
    rhs = oracle.compute_rhs(u, np.zeros_like(u), consts=c)
    s = (n - 1) // 12
    sl = slice(3 * s, n - 3 * s, s)   # >= 3 points from every face at n >= 13
    return np.abs(rhs[sl, sl, sl] - want[sl, sl, sl]).max(), np.abs(want[sl, sl, sl]).max()


def test_p7_full_nas_operator_converges_to_navier_stokes():
    """With every NAS constant as set_constants makes it (dssp included), the
    interior converges at second order to -div F + NS viscous + dx*U_xx."""
    e13, scale = full_error(13)
    e25, _ = full_error(25)
    e49, _ = full_error(49)
    assert 3.3 < e13 / e25 < 4.7, (e13, e25)
    assert 3.6 < e25 / e49 < 4.4, (e25, e49)
    assert e49 < 2e-3 * scale, (e49, scale)


@pytest.mark.parametrize("field,factor", [
    ("xxcon2", 1.5), ("xxcon3", 0.5), ("xxcon4", 2.0), ("xxcon5", 1.1),
    ("yycon2", 0.5), ("zzcon5", 0.9), ("dx3tx1", 2.0), ("dz5tz1", 0.5),
])
def test_p7_full_operator_mutants_do_not_converge(field, factor):
    def run(n):
        c = oracle.set_constants(n, n, n, 1.0)
        setattr(c, field, getattr(c, field) * factor)
        return full_error(n, c)
    e49, _ = run(49)
    ok49, _ = full_error(49)
    assert e49 > 2.0 * ok49, (field, e49, ok49)


def test_p7_aux_are_primitive_variables_and_sound_speed():
    """Step-0 aux on the gas state: rho_i = 1/rho, (us, vs, ws) = velocity,
    square = rho |v|^2 / 2, qs = |v|^2 / 2, and SP's speed = sqrt(gamma p / rho),
    the ideal-gas speed of sound (pins c1c2 = gamma (gamma - 1))."""
    g = np.linspace(0.0, 1.0, 11)
    z, y, x = np.meshgrid(g, g, g, indexing="ij")
    rho, u, v, w, p = primitives(x, y, z)
    a = oracle.compute_aux(conservative(x, y, z), naux=7)
    q = 0.5 * (u * u + v * v + w * w)
    for got, want in ((a[..., 0], 1.0 / rho), (a[..., 1], u), (a[..., 2], v), (a[..., 3], w),
                      (a[..., 4], rho * q), (a[..., 5], q), (a[..., 6], np.sqrt(GAMMA * p / rho))):
        np.testing.assert_allclose(got, want, rtol=1e-13, atol=1e-15)

"""Pins for the CPU oracle (oracle/) against what the mathematics fixes.

None of these retypes the oracle's loop nest.  Each checks the oracle against
an independent characterisation of NPB compute_rhs:

P1  constant field: every flux and second difference vanishes; the interior is
    dt*(f - dssp*c*(b_i + b_j + b_k)) with b = row sums of the dissipation
    operator, derived here from the textbook D = B^T B (not from the 5 cases).
P2  exact-solution residual: compute_rhs(exact_solution, exact_rhs) ~ 0, where
    nasgen.exact_rhs is NPB's independent formulation of the operator.
P4  linear-operator closed forms: fields for which the operator is linear are
    checked against second-difference / centred-difference / B^T B matrices
    built with numpy (catches wrong coefficient, axis, sign or stencil case).
P5  forcing affinity: rhs(u,f1) - rhs(u,f2) = dt (f1 - f2) inside, f1-f2 on faces.
P6  symmetry: swapping axes i<->j (and u2<->u3) or i<->k (with dz := dx)
    permutes the result the same way.
plus: set_constants closed forms, extent validation (reading c4).
"""
import os

import numpy as np
import pytest

import nasgen
import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ----------------------------------------------------------------------------
# Textbook operators along one axis of length n (rows 1..n-2 meaningful).
# ----------------------------------------------------------------------------
def second_difference(n):
    L = np.zeros((n, n))
    for i in range(1, n - 1):
        L[i, i - 1], L[i, i], L[i, i + 1] = 1.0, -2.0, 1.0
    return L


def centred_difference(n):
    C = np.zeros((n, n))
    for i in range(1, n - 1):
        C[i, i + 1], C[i, i - 1] = 1.0, -1.0
    return C


def dissipation_btb(n):
    """D = B^T B with B the second difference of the zero-extended interior
    field: the symmetric positive semi-definite fourth-order dissipation."""
    B = second_difference(n)
    B[:, 0] = 0.0
    B[:, n - 1] = 0.0
    D = B.T @ B
    D[0, :] = D[n - 1, :] = 0.0
    return D


def along(M, g, axis):
    """Apply matrix M along ``axis`` of the (k, j, i) field g."""
    return np.moveaxis(np.tensordot(M, g, axes=([1], [axis])), 0, axis)


def interior(a):
    return a[1:-1, 1:-1, 1:-1]


def faces_mask(nz, ny, nx):
    m = np.ones((nz, ny, nx), dtype=bool)
    m[1:-1, 1:-1, 1:-1] = False
    return m


# ----------------------------------------------------------------------------
def test_golden_dissipation_rows_match_btb():
    """The NAS 5-case stencil rows (golden) equal B^T B."""
    rows = np.loadtxt(os.path.join(GOLDEN, "dissipation_rows_n9.txt"))
    D = dissipation_btb(9)
    assert np.array_equal(rows, D[1:8, :])


def test_set_constants_closed_forms():
    for n in (6, 12, 36, 64, 102, 162):
        c = oracle.set_constants(n, n + 1, n + 2, 0.001)
        for ax, m in (("x", n), ("y", n + 1), ("z", n + 2)):
            t1, t2, t3 = getattr(c, f"t{ax}1"), getattr(c, f"t{ax}2"), getattr(c, f"t{ax}3")
            assert t1 == pytest.approx((m - 1) ** 2, rel=1e-14)
            assert t2 == pytest.approx((m - 1) / 2.0, rel=1e-14)
            assert t3 == pytest.approx(m - 1, rel=1e-14)
            cc = ax * 2
            assert getattr(c, f"{cc}con2") == pytest.approx(0.1 * (m - 1) ** 2, rel=1e-14)
            assert getattr(c, f"{cc}con1") == pytest.approx(0.1 * 4 / 3 * (m - 1) ** 2, rel=1e-14)
            assert getattr(c, f"{cc}con3") == pytest.approx(0.1 * (1 - 1.96) * (m - 1) ** 2, rel=1e-13)
            assert getattr(c, f"{cc}con4") == pytest.approx(0.1 / 6 * (m - 1) ** 2, rel=1e-14)
            assert getattr(c, f"{cc}con5") == pytest.approx(0.1 * 1.96 * (m - 1) ** 2, rel=1e-14)
        assert c.dssp == 0.25
        assert c.dx1tx1 == pytest.approx(0.75 * (n - 1) ** 2, rel=1e-14)
        assert c.dz5tz1 == pytest.approx(1.0 * (n + 1) ** 2, rel=1e-14)


@pytest.mark.parametrize("n", [4, 5])
def test_rejects_small_extents(n):
    u = np.ones((n, 8, 8, 5))
    with pytest.raises(ValueError):
        oracle.compute_rhs(u, u, dt=0.01)
    u = np.ones((8, 8, n, 5))
    with pytest.raises(ValueError):
        oracle.compute_rhs(u, u, dt=0.01)


@pytest.mark.parametrize("shape", [(6, 6, 6), (7, 7, 7), (9, 8, 7), (12, 12, 12)])
def test_p1_constant_field(shape):
    nz, ny, nx = shape
    rng = np.random.default_rng(11)
    cvec = np.array([2.5, 0.75, -1.25, 1.5, 9.0])
    u = np.broadcast_to(cvec, (nz, ny, nx, 5)).copy()
    f = rng.uniform(-3, 3, size=(nz, ny, nx, 5))
    dt = 0.0125
    r = oracle.compute_rhs(u, f, dt=dt)
    c = oracle.set_constants(nx, ny, nz, dt)
    bx = dissipation_btb(nx).sum(axis=1)
    by = dissipation_btb(ny).sum(axis=1)
    bz = dissipation_btb(nz).sum(axis=1)
    b = bz[:, None, None] + by[None, :, None] + bx[None, None, :]
    expect = dt * (f - c.dssp * cvec[None, None, None, :] * b[..., None])
    assert np.allclose(interior(r), interior(expect), rtol=0, atol=1e-14)
    fm = faces_mask(nz, ny, nx)
    assert np.array_equal(r[fm], f[fm])


@pytest.mark.parametrize("bench,cls", [("BT", "S"), ("SP", "W"), ("BT", "W"), ("BT", "A")])
def test_p2_exact_solution_residual(bench, cls):
    inp = nasgen.make_class(bench, cls, A=0.0)
    r = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=4)
    assert np.abs(interior(r)).max() <= 1e-13, np.abs(interior(r)).max()
    fm = faces_mask(inp.nz, inp.ny, inp.nx)
    assert np.array_equal(r[fm], inp.forcing[fm])
    # The forcing is O(10): a dropped or mis-signed term would leave O(1e-3..10).
    assert np.abs(inp.forcing).max() > 10


def test_p2_exact_solution_residual_noncubic():
    nx, ny, nz = 14, 9, 11
    u = nasgen.exact_grid(nx, ny, nz)
    f = nasgen.exact_rhs(nx, ny, nz)
    r = oracle.compute_rhs(u, f, dt=0.003)
    assert np.abs(interior(r)).max() <= 1e-13


def test_p2_residual_detects_perturbation():
    """Sanity of the pin itself: perturb one u value -> residual is O(1)."""
    nx = 12
    u = nasgen.exact_grid(nx, nx, nx)
    f = nasgen.exact_rhs(nx, nx, nx)
    u[5, 6, 7, 2] *= 1.0 + 1e-6
    r = oracle.compute_rhs(u, f, dt=1.0)
    assert np.abs(interior(r)).max() > 1e-6


@pytest.mark.parametrize("shape", [(7, 8, 9), (11, 6, 13)])
def test_p4_energy_only_linear_operator(shape):
    """u1=1, u2=u3=u4=0, u5=g: every term is linear in g (App. A with
    us=vs=ws=square=qs=0, rho_i=1)."""
    nz, ny, nx = shape
    rng = np.random.default_rng(5)
    g = rng.uniform(1.0, 2.0, size=(nz, ny, nx))
    u = np.zeros((nz, ny, nx, 5))
    u[..., 0] = 1.0
    u[..., 4] = g
    f = rng.uniform(-1, 1, size=(nz, ny, nx, 5))
    dt = 0.02
    c = oracle.set_constants(nx, ny, nz, dt)
    r = oracle.compute_rhs(u, f, dt=dt)

    Lx, Ly, Lz = (second_difference(n) for n in (nx, ny, nz))
    Cx, Cy, Cz = (centred_difference(n) for n in (nx, ny, nz))
    Dx, Dy, Dz = (dissipation_btb(n) for n in (nx, ny, nz))
    one = np.ones_like(g)
    diss = lambda a: along(Dx, a, 2) + along(Dy, a, 1) + along(Dz, a, 0)

    e = np.empty_like(f)
    e[..., 0] = dt * (f[..., 0] - c.dssp * diss(one))
    e[..., 1] = dt * (f[..., 1] - c.tx2 * c.c2 * along(Cx, g, 2))
    e[..., 2] = dt * (f[..., 2] - c.ty2 * c.c2 * along(Cy, g, 1))
    e[..., 3] = dt * (f[..., 3] - c.tz2 * c.c2 * along(Cz, g, 0))
    e[..., 4] = dt * (f[..., 4]
                      + (c.dx5tx1 + c.xxcon5) * along(Lx, g, 2)
                      + (c.dy5ty1 + c.yycon5) * along(Ly, g, 1)
                      + (c.dz5tz1 + c.zzcon5) * along(Lz, g, 0)
                      - c.dssp * diss(g))
    scale = dt * 200.0 * max(nx, ny, nz) ** 2
    assert np.allclose(interior(r), interior(e), rtol=0, atol=1e-13 * scale)
    fm = faces_mask(nz, ny, nx)
    assert np.array_equal(r[fm], f[fm])


@pytest.mark.parametrize("mom", [1, 2, 3])
def test_p4_continuity_flux(mom):
    """u1 = const, one momentum component = g: rhs1 is the centred difference
    of that momentum along its own axis (continuity equation) minus the
    dissipation of the constant density."""
    nz, ny, nx = 9, 10, 11
    rng = np.random.default_rng(100 + mom)
    g = rng.uniform(-1.0, 1.0, size=(nz, ny, nx))
    u = np.zeros((nz, ny, nx, 5))
    u[..., 0] = 2.0
    u[..., mom] = g
    u[..., 4] = 6.0
    f = rng.uniform(-1, 1, size=(nz, ny, nx, 5))
    dt = 0.05
    c = oracle.set_constants(nx, ny, nz, dt)
    r = oracle.compute_rhs(u, f, dt=dt)
    axis = {1: 2, 2: 1, 3: 0}[mom]
    t2 = {1: c.tx2, 2: c.ty2, 3: c.tz2}[mom]
    C = centred_difference(u.shape[axis])
    D = [dissipation_btb(n) for n in (nx, ny, nz)]
    two = 2.0 * np.ones_like(g)
    diss = along(D[0], two, 2) + along(D[1], two, 1) + along(D[2], two, 0)
    e1 = dt * (f[..., 0] - t2 * along(C, g, axis) - c.dssp * diss)
    assert np.allclose(interior(r[..., 0]), interior(e1), rtol=0, atol=1e-14 * 100)


def test_p5_forcing_affinity(inputs_cache):
    inp = inputs_cache(10, 11, 12, seed=2, dt=0.004)
    rng = np.random.default_rng(3)
    f2 = inp.forcing + rng.uniform(-1, 1, size=inp.forcing.shape)
    r1 = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt)
    r2 = oracle.compute_rhs(inp.u, f2, dt=inp.dt)
    d = r1 - r2
    e = inp.dt * (inp.forcing - f2)
    assert np.allclose(interior(d), interior(e), rtol=0, atol=1e-15 * 50)
    fm = faces_mask(inp.nz, inp.ny, inp.nx)
    assert np.array_equal(d[fm], (inp.forcing - f2)[fm])


def test_p6_symmetry_i_j(inputs_cache):
    n = 10
    inp = inputs_cache(n, n, 13, seed=3, dt=0.002)
    dt = inp.dt
    r = oracle.compute_rhs(inp.u, inp.forcing, dt=dt)
    perm = [0, 2, 1, 3, 4]
    uT = np.ascontiguousarray(inp.u.transpose(0, 2, 1, 3)[..., perm])
    fT = np.ascontiguousarray(inp.forcing.transpose(0, 2, 1, 3)[..., perm])
    rT = oracle.compute_rhs(uT, fT, dt=dt)
    back = rT.transpose(0, 2, 1, 3)[..., perm]
    scale = np.abs(r).max()
    assert np.allclose(back, r, rtol=0, atol=1e-13 * max(scale, 1.0))


def test_p6_symmetry_i_k(inputs_cache):
    n = 9
    inp = inputs_cache(n, 11, n, seed=4, dt=0.002)
    dt = inp.dt
    c = oracle.set_constants(n, 11, n, dt)
    # NAS uses dz = 1.0 but dx = 0.75; make the operator i<->k symmetric.
    for m in range(1, 6):
        setattr(c, f"dz{m}tz1", getattr(c, f"dx{m}tx1"))
    r = oracle.compute_rhs(inp.u, inp.forcing, consts=c)
    perm = [0, 3, 2, 1, 4]
    uT = np.ascontiguousarray(inp.u.transpose(2, 1, 0, 3)[..., perm])
    fT = np.ascontiguousarray(inp.forcing.transpose(2, 1, 0, 3)[..., perm])
    rT = oracle.compute_rhs(uT, fT, consts=c)
    back = rT.transpose(2, 1, 0, 3)[..., perm]
    scale = np.abs(r).max()
    assert np.allclose(back, r, rtol=0, atol=1e-13 * max(scale, 1.0))


def test_thread_count_invariance(inputs_cache):
    inp = inputs_cache(16, 14, 12, seed=1, dt=0.001)
    r1 = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=1)
    r4 = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=4)
    assert np.array_equal(r1, r4)


def test_generator_determinism():
    a = nasgen.make_inputs(8, 9, 10, seed=7)
    b = nasgen.make_inputs(8, 9, 10, seed=7)
    c = nasgen.make_inputs(8, 9, 10, seed=8)
    assert np.array_equal(a.u, b.u) and np.array_equal(a.forcing, b.forcing)
    assert not np.array_equal(a.u, c.u)
    xi = nasgen.uniform_pm1(1, 0, (1000,))
    assert xi.min() >= -1.0 and xi.max() < 1.0 and abs(xi.mean()) < 0.1

"""GPU parity of the SURVEY §8(f) f1 outputs through the C ABI: the step-0
auxiliary fields written alongside rhs (safara_rhs_aux / _slab_aux) and the
rhs_norm numerator (safara_rhs_sumsq), against the CPU oracle
(oracle.compute_aux / oracle.rhs_sumsq, pinned in test_oracle_aux_pins.py).

Bars: STRICT aux and rhs bit-identical; production within
|g - o| <= 1e-12 |o| + 1e-14 (reading c5); sums of squares within 1e-12
relative (the reduction order differs from the Fortran loop order).
"""
import ctypes

import numpy as np
import pytest
import torch

import nasgen
import oracle
import paper_conf_icpp_tiankexc16_b200 as sr

pytestmark = pytest.mark.gpu

RTOL, ATOL = 1e-12, 1e-14


@pytest.fixture(scope="module", autouse=True)
def _init():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    sr.init(0)


def assert_tol(g, o):
    err = np.abs(g - o)
    bound = RTOL * np.abs(o) + ATOL
    bad = err > bound
    assert not bad.any(), (f"{bad.sum()} elements out of tolerance; worst ratio "
                           f"{(err / bound).max():.3g}")


def run_aux(inp, naux, strict):
    nz, ny, nx, _ = inp.u.shape
    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    dr = torch.full_like(du, float("nan"))
    da = torch.full((nz, naux, ny, sr.pitch(nx)), float("nan"), dtype=torch.float64,
                    device="cuda")
    c = sr.coeffs_nas(nx, ny, nz, inp.dt)
    n0 = sr.launch_count()
    sr.rhs_aux(du, df, dr, da, nx, c, strict=strict)
    torch.cuda.synchronize()
    assert sr.launch_count() == n0 + 1
    return sr.unpack(dr, nx), sr.unpack_aux(da, nx)


CASES = [("BT", "S", None), ("SP", "W", None), (None, None, (9, 13, 37)), (None, None, (40, 7, 11))]


@pytest.mark.parametrize("bench,cls,shape", CASES)
@pytest.mark.parametrize("naux", [6, 7])
@pytest.mark.parametrize("strict", [True, False])
def test_aux_parity(bench, cls, shape, naux, strict):
    if bench:
        inp = nasgen.make_class(bench, cls, seed=1, B=1e-2)
    else:
        inp = nasgen.make_inputs(*shape, seed=7, dt=0.001)
    g_rhs, g_aux = run_aux(inp, naux, strict)
    o_rhs = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=8)
    o_aux = oracle.compute_aux(inp.u, naux, dt=inp.dt)
    assert not np.isnan(g_aux).any(), "some aux point was not written"
    if strict:
        assert np.array_equal(g_rhs, o_rhs)
        assert np.array_equal(g_aux, o_aux)
    else:
        assert_tol(g_rhs, o_rhs)
        assert_tol(g_aux, o_aux)


@pytest.mark.parametrize("p", [2, 3])
@pytest.mark.parametrize("split", [False, True])
def test_aux_slabs(p, split):
    """z-slab aux (ghosted u, global-k faces) reproduces the full-grid aux."""
    nx, ny, nz = 19, 14, 23
    inp = nasgen.make_inputs(nx, ny, nz, seed=8, dt=0.001)
    c = sr.coeffs_nas(nx, ny, nz, inp.dt)
    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    aux = torch.full((nz, 7, ny, sr.pitch(nx)), float("nan"), dtype=torch.float64, device="cuda")
    out = torch.full_like(du, float("nan"))
    base, rem = divmod(nz, p)
    k0 = 0
    for r in range(p):
        nzl = base + (1 if r < rem else 0)
        us = torch.zeros((nzl + 4,) + tuple(du.shape[1:]), dtype=torch.float64, device="cuda")
        lo, hi = max(k0 - 2, 0), min(k0 + nzl + 2, nz)
        us[lo - (k0 - 2):hi - (k0 - 2)] = du[lo:hi]
        fs = df[k0:k0 + nzl].contiguous()
        rs = torch.full_like(fs, float("nan"))
        a_s = torch.full((nzl, 7, ny, sr.pitch(nx)), float("nan"), dtype=torch.float64,
                         device="cuda")
        parts = ([sr.SAFARA_PART_INTERIOR, sr.SAFARA_PART_EDGE] if split
                 else [sr.SAFARA_PART_ALL])
        for part in parts:
            sr.rhs_slab_aux(us, fs, rs, a_s, nx, nz, k0, c, part=part, strict=True)
        out[k0:k0 + nzl] = rs
        aux[k0:k0 + nzl] = a_s
        k0 += nzl
    torch.cuda.synchronize()
    assert np.array_equal(sr.unpack(out, nx),
                          oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=8))
    assert np.array_equal(sr.unpack_aux(aux, nx), oracle.compute_aux(inp.u, 7, dt=inp.dt))


def test_aux_sp_native_layout():
    """aux with components outermost follows u's [m][k][j][i] (plane stride sk)."""
    inp = nasgen.make_inputs(30, 22, 14, seed=4, dt=0.002)
    nz, ny, nx, _ = inp.u.shape
    sy = sr.pitch(nx)
    d = sr.Dims(nx, ny, nz, sy, sy * ny * nz, sy * ny)

    def to_sp(a, ncomp):
        t = torch.zeros((ncomp, nz, ny, sy), dtype=torch.float64)
        t[..., :nx] = torch.from_numpy(a).permute(3, 0, 1, 2)
        return t.cuda().contiguous()

    du, df = to_sp(inp.u, 5), to_sp(inp.forcing, 5)
    dr = torch.full_like(du, float("nan"))
    da = torch.full((7, nz, ny, sy), float("nan"), dtype=torch.float64, device="cuda")
    c = sr.coeffs_nas(nx, ny, nz, inp.dt)
    sr._abi.check(sr._abi.lib().safara_rhs_aux(du.data_ptr(), df.data_ptr(), dr.data_ptr(),
                                          da.data_ptr(), 7, ctypes.byref(d), ctypes.byref(c),
                                          sr.SAFARA_FLAG_STRICT, None), "safara_rhs_aux")
    torch.cuda.synchronize()
    g = da[..., :nx].permute(1, 2, 3, 0).cpu().numpy()
    assert np.array_equal(g, oracle.compute_aux(inp.u, 7, dt=inp.dt))


def test_aux_error_paths():
    L = sr._abi.lib()
    nx = ny = nz = 12
    d = sr.canonical_dims(nx, ny, nz)
    c = sr.coeffs_nas(nx, ny, nz, 0.01)
    u = torch.zeros((nz, 5, ny, sr.pitch(nx)), dtype=torch.float64, device="cuda")
    f, r = torch.zeros_like(u), torch.zeros_like(u)
    a = torch.zeros((nz, 7, ny, sr.pitch(nx)), dtype=torch.float64, device="cuda")
    args = lambda aux, naux: (u.data_ptr(), f.data_ptr(), r.data_ptr(), aux, naux,
                              ctypes.byref(d), ctypes.byref(c), 0, None)
    assert L.safara_rhs_aux(*args(a.data_ptr(), 5)) == -1          # naux
    assert L.safara_rhs_aux(*args(None, 6)) == -1                   # NULL aux
    assert L.safara_rhs_aux(*args(r.data_ptr(), 6)) == -1           # aux aliases rhs
    assert L.safara_rhs_aux(*args(a.data_ptr() + 4, 6)) == -4       # misaligned
    assert L.safara_rhs_aux(*args(a.data_ptr(), 7)) == 0


@pytest.mark.parametrize("bench,cls", [("BT", "S"), ("SP", "W"), ("BT", "A")])
def test_sumsq_full_grid(bench, cls):
    inp = nasgen.make_class(bench, cls, seed=3, B=1e-2)
    nz, ny, nx, _ = inp.u.shape
    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    dr = torch.empty_like(du)
    sr.rhs(du, df, dr, nx, sr.coeffs_nas(nx, ny, nz, inp.dt), strict=True)
    n0 = sr.launch_count()
    g = sr.rhs_sumsq(dr, nx).cpu().numpy()
    assert sr.launch_count() == n0 + 2
    o = oracle.rhs_sumsq(oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=8))
    np.testing.assert_allclose(g, o, rtol=1e-12, atol=0)
    # deterministic: the same bits on a second call
    assert np.array_equal(g, sr.rhs_sumsq(dr, nx).cpu().numpy())
    rms = sr.rhs_norm(dr, nx)
    np.testing.assert_allclose(rms, np.sqrt(o / (nx - 2) / (ny - 2) / (nz - 2)), rtol=1e-12)


def test_sumsq_slabs_add_up():
    """Per-slab sums (interior planes only, global k) add up to the grid's."""
    inp = nasgen.make_inputs(17, 15, 29, seed=9, dt=0.001)
    nz, ny, nx, _ = inp.u.shape
    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    dr = torch.empty_like(du)
    sr.rhs(du, df, dr, nx, sr.coeffs_nas(nx, ny, nz, inp.dt))
    total = sr.rhs_sumsq(dr, nx).cpu().numpy()
    parts = []
    for k0, k1 in ((0, 7), (7, 19), (19, 29)):
        parts.append(sr.rhs_sumsq(dr[k0:k1].contiguous(), nx, nz=nz, k0=k0).cpu().numpy())
    np.testing.assert_allclose(np.sum(parts, axis=0), total, rtol=1e-13)


@pytest.mark.parametrize("strict", [True, False])
def test_aux_analytic_gas_state(strict):
    """P7's analytic gas state (tests/test_oracle_euler_pins.py): the GPU aux
    fields against the oracle (bitwise in STRICT) and SP speed against the
    ideal-gas sound speed sqrt(gamma p / rho)."""
    from types import SimpleNamespace
    from test_oracle_euler_pins import GAMMA, conservative, primitives
    nz, ny, nx = 21, 17, 45
    z, y, x = np.meshgrid(np.linspace(0, 1, nz), np.linspace(0, 1, ny),
                          np.linspace(0, 1, nx), indexing="ij")
    u = conservative(x, y, z)
    inp = SimpleNamespace(u=u, forcing=0.5 * u, dt=1e-3)
    g_rhs, g_aux = run_aux(inp, 7, strict)
    o_aux = oracle.compute_aux(u, naux=7, dt=inp.dt)
    o_rhs = oracle.compute_rhs(u, inp.forcing, dt=inp.dt, threads=8)
    if strict:
        assert np.array_equal(g_aux, o_aux) and np.array_equal(g_rhs, o_rhs)
    else:
        assert_tol(g_aux, o_aux)
        assert_tol(g_rhs, o_rhs)
    rho, _, _, _, p = primitives(x, y, z)
    np.testing.assert_allclose(g_aux[..., 6], np.sqrt(GAMMA * p / rho), rtol=1e-13)


# ---- round 2: rhs_norm fused into the store epilogue (safara_rhs_fused) ----

@pytest.mark.parametrize("bench,cls", [("BT", "W"), ("BT", "C")])
@pytest.mark.parametrize("with_aux", [False, True])
def test_fused_norm_matches_oracle(bench, cls, with_aux):
    """NPB rhs_norm accumulated in the pass (per-thread sums, CTA partials,
    one finishing launch) equals the oracle's norm of the oracle's rhs; rhs and
    aux are unchanged by the fusion (STRICT bitwise)."""
    inp = nasgen.make_class(bench, cls, seed=1, B=1e-2)
    nz, ny, nx, _ = inp.u.shape
    c = sr.coeffs_nas(nx, ny, nz, inp.dt)
    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    dr = torch.full_like(du, float("nan"))
    da = sr.empty_aux(nx, ny, nz, sr.SAFARA_AUX_BT) if with_aux else None
    n0 = sr.launch_count()
    rms = sr.rhs_fused(du, df, dr, nx, c, aux=da, rms=True, strict=True)
    torch.cuda.synchronize()
    # class C: the warp-specialised kernel finishes the norm in its last CTA
    # (one launch); small grids take the two-pass path (3 launches)
    assert sr.launch_count() - n0 == (1 if cls == "C" else 3)
    o = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=8)
    assert np.array_equal(sr.unpack(dr, nx), o)
    if with_aux:
        assert np.array_equal(sr.unpack_aux(da, nx), oracle.compute_aux(inp.u, 6, dt=inp.dt))
    want = np.sqrt(oracle.rhs_sumsq(o) / ((nx - 2) * (ny - 2) * (nz - 2)))
    np.testing.assert_allclose(rms.cpu().numpy(), want, rtol=1e-13, atol=0)
    # production: same contract (rhs within c5), norm to 1e-13 of the oracle's
    rms2 = sr.rhs_fused(du, df, dr, nx, c, aux=da, rms=True)
    torch.cuda.synchronize()
    np.testing.assert_allclose(rms2.cpu().numpy(), want, rtol=1e-12, atol=0)


def test_fused_norm_general_coefficients_falls_back_to_two_pass():
    """General (non-NAS) coefficients: no fused-norm kernel instance; the
    library runs the two-pass norm (3 launches) with the same result."""
    inp = nasgen.make_class("BT", "W", seed=2)
    nz, ny, nx, _ = inp.u.shape
    c = sr.coeffs_nas(nx, ny, nz, inp.dt)
    c.dxt[2] *= 1.01      # dx3 != dx1: the general-coefficient kernel
    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    dr = torch.empty_like(du)
    n0 = sr.launch_count()
    rms = sr.rhs_fused(du, df, dr, nx, c, rms=True, strict=True)
    torch.cuda.synchronize()
    assert sr.launch_count() - n0 == 3
    g = sr.unpack(dr, nx)
    want = np.sqrt(oracle.rhs_sumsq(g) / ((nx - 2) * (ny - 2) * (nz - 2)))
    np.testing.assert_allclose(rms.cpu().numpy(), want, rtol=1e-13, atol=0)


@pytest.mark.parametrize("p", [2, 3, 8])
def test_slab_norms_sum_to_full_grid_norm(p):
    """z-slab partial sums (safara_rhs_sumsq per slab, the numerators the
    sharded all-reduce adds) give the full-grid rhs_norm to 1e-13."""
    from paper_conf_icpp_tiankexc16_b200 import dist as sd
    inp = nasgen.make_class("BT", "A", seed=1, B=1e-2)
    nz, ny, nx, _ = inp.u.shape
    c = sr.coeffs_nas(nx, ny, nz, inp.dt)
    ug, fg = sr.pack(inp.u, device="cpu"), sr.pack(inp.forcing, device="cpu")
    tot = np.zeros(5)
    for r in range(p):
        s = sd.make_slab(ug, fg, nx, r, p, device="cuda")
        k0, nzl = sd.partition(nz, p)[r]
        # ghosts from the global field (what the exchange delivers)
        lo, hi = max(0, k0 - 2), min(nz, k0 + nzl + 2)
        s.u[lo - (k0 - 2):hi - (k0 - 2)] = ug[lo:hi].cuda()
        sr.rhs_slab(s.u, s.forcing, s.rhs, nx, nz, k0, c, strict=True)
        tot += sr.rhs_sumsq(s.rhs, nx, nz=nz, k0=k0).cpu().numpy()
    torch.cuda.synchronize()
    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    dr = torch.empty_like(du)
    full = sr.rhs_fused(du, df, dr, nx, c, rms=True, strict=True).cpu().numpy()
    npts = (nx - 2) * (ny - 2) * (nz - 2)
    np.testing.assert_allclose(np.sqrt(tot / npts), full, rtol=1e-13, atol=0)

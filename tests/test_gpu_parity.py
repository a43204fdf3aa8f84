"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bar: STRICT variant bit-identical to the oracle; production
variant within |g - o| <= 1e-12 |o| + 1e-14 elementwise (BASELINE.json
north_star, reading c5).  Inputs: nasgen (exact solution x (1 + 1e-3 noise),
forcing = exact_rhs [+ noise]), identical on both sides.
"""
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


def gpu_rhs(u, f, dt, strict, nx=None):
    nz, ny, nx_, _ = u.shape
    nx = nx_ if nx is None else nx
    du, df = sr.pack(u), sr.pack(f)
    dr = torch.full_like(du, float("nan"))
    c = sr.coeffs_nas(nx, ny, nz, dt)
    n0 = sr.launch_count()
    sr.rhs(du, df, dr, nx, c, strict=strict)
    torch.cuda.synchronize()
    assert sr.launch_count() == n0 + 1
    return sr.unpack(dr, nx)


def assert_tol(g, o):
    err = np.abs(g - o)
    bound = RTOL * np.abs(o) + ATOL
    bad = err > bound
    assert not bad.any(), (f"{bad.sum()} elements out of tolerance; worst ratio "
                           f"{(err / bound).max():.3g}")


def oracle_rhs(inp):
    return oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=8)


SMALL = [("BT", "S"), ("SP", "W"), ("BT", "W"), ("BT", "A")]


@pytest.mark.parametrize("bench,cls", SMALL)
def test_strict_bitwise_classes(bench, cls):
    inp = nasgen.make_class(bench, cls, seed=1, B=1e-2)
    o = oracle_rhs(inp)
    g = gpu_rhs(inp.u, inp.forcing, inp.dt, strict=True)
    assert np.array_equal(g, o), f"max |g-o| = {np.abs(g - o).max():.3g}"


@pytest.mark.parametrize("shape", [(6, 6, 6), (7, 7, 7), (9, 13, 37), (17, 29, 37),
                                   (11, 70, 41), (8, 12, 66), (23, 15, 100)])
def test_strict_bitwise_ragged(shape):
    nz, ny, nx = shape
    inp = nasgen.make_inputs(nx, ny, nz, seed=2, B=1e-2, dt=0.003)
    o = oracle_rhs(inp)
    g = gpu_rhs(inp.u, inp.forcing, inp.dt, strict=True)
    assert np.array_equal(g, o), f"max |g-o| = {np.abs(g - o).max():.3g}"


@pytest.mark.parametrize("bench,cls", SMALL + [("SP", "B"), ("BT", "C")])
def test_fast_within_tolerance(bench, cls):
    inp = nasgen.make_class(bench, cls, seed=3)
    o = oracle_rhs(inp)
    g = gpu_rhs(inp.u, inp.forcing, inp.dt, strict=False)
    assert_tol(g, o)
    faces = np.ones(o.shape[:3], dtype=bool)
    faces[1:-1, 1:-1, 1:-1] = False
    assert np.array_equal(g[faces], inp.forcing[faces])


@pytest.mark.parametrize("bench,cls", [("SP", "B"), ("BT", "C")])
def test_strict_bitwise_large(bench, cls):
    inp = nasgen.make_class(bench, cls, seed=1)
    o = oracle_rhs(inp)
    g = gpu_rhs(inp.u, inp.forcing, inp.dt, strict=True)
    assert np.array_equal(g, o)


@pytest.mark.parametrize("strict", [True, False])
def test_general_coefficients(strict):
    """Non-NAS coefficients (dX1..dX5 not all equal) take the general kernel
    instead of the uniform-d1 specialisation; both sides get the same values."""
    inp = nasgen.make_inputs(40, 27, 19, seed=8, B=1e-2, dt=0.002)
    nz, ny, nx, _ = inp.u.shape
    oc = oracle.set_constants(nx, ny, nz, inp.dt)
    c = sr.coeffs_nas(nx, ny, nz, inp.dt)
    for m, f in enumerate((1.0, 1.1, 0.9, 1.3, 0.7)):
        setattr(oc, f"dx{m + 1}tx1", getattr(oc, f"dx{m + 1}tx1") * f)
        setattr(oc, f"dz{m + 1}tz1", getattr(oc, f"dz{m + 1}tz1") * (2.0 - f))
        c.dxt[m] = getattr(oc, f"dx{m + 1}tx1")
        c.dzt[m] = getattr(oc, f"dz{m + 1}tz1")
    o = oracle.compute_rhs(inp.u, inp.forcing, consts=oc)
    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    dr = torch.full_like(du, float("nan"))
    sr.rhs(du, df, dr, nx, c, strict=strict)
    torch.cuda.synchronize()
    g = sr.unpack(dr, nx)
    if strict:
        assert np.array_equal(g, o)
    else:
        assert_tol(g, o)


def test_exact_solution_residual_gpu():
    inp = nasgen.make_class("BT", "A", A=0.0)
    g = gpu_rhs(inp.u, inp.forcing, inp.dt, strict=False)
    assert np.abs(g[1:-1, 1:-1, 1:-1]).max() < 1e-13


def test_sp_native_layout_descriptor():
    """`dim` with another stride order: SP's native u(i,j,k,m) = [m][k][j][i]."""
    inp = nasgen.make_inputs(30, 22, 14, seed=4, dt=0.002)
    nz, ny, nx, _ = inp.u.shape
    sy = sr.pitch(nx)
    d = sr.Dims(nx, ny, nz, sy, sy * ny * nz, sy * ny)

    def to_sp(a):
        t = torch.zeros((5, nz, ny, sy), dtype=torch.float64)
        t[..., :nx] = torch.from_numpy(a).permute(3, 0, 1, 2)
        return t.cuda().contiguous()

    du, df = to_sp(inp.u), to_sp(inp.forcing)
    dr = torch.full_like(du, float("nan"))
    c = sr.coeffs_nas(nx, ny, nz, inp.dt)
    sr.rhs(du, df, dr, nx, c, strict=True, dims=d)
    torch.cuda.synchronize()
    g = dr[..., :nx].permute(1, 2, 3, 0).cpu().numpy()
    assert np.array_equal(g, oracle_rhs(inp))


@pytest.mark.parametrize("nz,p", [(12, 2), (36, 3), (64, 2), (41, 4), (102, 8), (24, 8)])
@pytest.mark.parametrize("split", [False, True])
@pytest.mark.parametrize("strict", [True, False])
def test_slab_decomposition(nz, p, split, strict):
    """z-slabs computed one after another on one GPU (ghost planes copied from
    the global array) reproduce the single-GPU result: bit for bit in STRICT
    (no contraction anywhere), within the parity tolerance in production mode
    (the compiler may contract differently in the code paths that handle the
    first planes of a slab)."""
    nx, ny = 21, 18
    inp = nasgen.make_inputs(nx, ny, nz, seed=5, dt=0.001)
    c = sr.coeffs_nas(nx, ny, nz, inp.dt)
    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    ref = torch.full_like(du, float("nan"))
    sr.rhs(du, df, ref, nx, c, strict=strict)
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
        if split:
            sr.rhs_slab(us, fs, rs, nx, nz, k0, c, part=sr.SAFARA_PART_INTERIOR, strict=strict)
            sr.rhs_slab(us, fs, rs, nx, nz, k0, c, part=sr.SAFARA_PART_EDGE, strict=strict)
        else:
            sr.rhs_slab(us, fs, rs, nx, nz, k0, c, part=sr.SAFARA_PART_ALL, strict=strict)
        out[k0:k0 + nzl] = rs
        k0 += nzl
    torch.cuda.synchronize()
    a, b = sr.unpack(out, nx), sr.unpack(ref, nx)
    if strict:
        assert np.array_equal(a, b)
    else:
        assert_tol(a, b)
        assert_tol(a, oracle_rhs(inp))


@pytest.mark.parametrize("nchunks", [1, 3, 8])
def test_host_e2e_path(nchunks):
    inp = nasgen.make_class("SP", "W", seed=6)
    nz, ny, nx, _ = inp.u.shape
    hu, hf = sr.pack(inp.u, pin=True), sr.pack(inp.forcing, pin=True)
    hr = torch.zeros_like(hu).pin_memory()
    du, df, dr = (torch.empty(hu.shape, dtype=torch.float64, device="cuda") for _ in range(3))
    c = sr.coeffs_nas(nx, ny, nz, inp.dt)
    n0 = sr.launch_count()
    sr.rhs_host(hu, hf, hr, du, df, dr, nx, c, strict=True, nchunks=nchunks)
    torch.cuda.synchronize()
    assert sr.launch_count() - n0 == min(nchunks, nz // 4)
    assert np.array_equal(sr.unpack(hr, nx), oracle_rhs(inp))


def test_error_paths():
    nx = ny = nz = 12
    c = sr.coeffs_nas(nx, ny, nz, 0.01)
    du = sr.empty_field(nx, ny, nz)
    df = sr.empty_field(nx, ny, nz)
    dr = sr.empty_field(nx, ny, nz)
    with pytest.raises(sr.SafaraError) as e:      # rhs aliases u
        sr.rhs(du, df, du, nx, c)
    assert e.value.code == -1
    flat = torch.empty(du.numel() + 1, dtype=torch.float64, device="cuda")
    mis = flat[1:].view(du.shape)                 # 8-byte, not 16-byte, aligned
    with pytest.raises(sr.SafaraError) as e:
        sr.rhs(mis, df, dr, nx, c)
    assert e.value.code == -4
    small = sr.empty_field(5, 5, 5)
    with pytest.raises(sr.SafaraError) as e:
        sr.rhs(small, small.clone(), small.clone(), 5, c)
    assert e.value.code == -2
    # slab with a single owned plane
    us = sr.empty_field(nx, ny, 5)
    fs = sr.empty_field(nx, ny, 1)
    with pytest.raises(sr.SafaraError) as e:
        sr.rhs_slab(us, fs, fs.clone(), nx, nz, 3, c)
    assert e.value.code == -2


def test_kernel_info_zero_spill():
    """The production kernel (the bench's) has no local memory at all; the
    STRICT validation variant of the warp-specialised kernel (no FMA
    contraction: more live temporaries at the 160-register consumer budget)
    spills a few words outside the hot loads (profiles/ptxas_r02.txt)."""
    for strict in (False, True):
        k = sr.kernel_info(strict)
        assert k["local_bytes"] == 0 if not strict else k["local_bytes"] <= 64
        assert k["ctas_per_sm"] >= 1
        assert k["regs_per_thread"] <= 255


@pytest.mark.parametrize("shape", [(49, 49, 49), (37, 45, 61)])
def test_analytic_navier_stokes_field(shape):
    """P7's smooth analytic gas state (O(1) gradients in every component, unlike
    the exact-solution x noise inputs).  STRICT: bitwise.  Production: with
    zero forcing and dt = 1 the interior is a sum of O(tx1 |U|) ~ 1e3 terms
    cancelling to O(1), so no contraction order meets an elementwise relative
    bound near the zeros (measured: up to 35x it); the bound there is
    normwise per component (measured <= 7e-14).  With a NAS-scaled forcing and
    dt (forcing = u/2, dt = 1e-3) the elementwise c5 bound holds (0.12 of it)."""
    from test_oracle_euler_pins import conservative
    nz, ny, nx = shape
    z, y, x = np.meshgrid(np.linspace(0, 1, nz), np.linspace(0, 1, ny),
                          np.linspace(0, 1, nx), indexing="ij")
    u = conservative(x, y, z)
    f = np.zeros_like(u)
    o = oracle.compute_rhs(u, f, dt=1.0, threads=8)
    assert np.array_equal(gpu_rhs(u, f, 1.0, strict=True), o)
    g = gpu_rhs(u, f, 1.0, strict=False)
    for m in range(5):
        assert np.abs(g[..., m] - o[..., m]).max() <= RTOL * np.abs(o[..., m]).max()
    f = 0.5 * u
    o = oracle.compute_rhs(u, f, dt=1e-3, threads=8)
    assert np.array_equal(gpu_rhs(u, f, 1e-3, strict=True), o)
    assert_tol(gpu_rhs(u, f, 1e-3, strict=False), o)


@pytest.mark.xfail(strict=True, reason="production variant on the cancellation-dominated "
                   "P7 state (zero forcing, dt = 1): the elementwise c5 bound is missed by up "
                   "to ~35x at near-zero outputs (DESIGN.md c5; the normwise bound holds)")
def test_analytic_state_production_elementwise_gap():
    """Records the gap the header states (include/safara.h, safara_rhs): on
    O(1e3) terms cancelling to O(1), production is held to the normwise bound
    only.  Strict xfail: if a change closes the gap, this test says so."""
    from test_oracle_euler_pins import conservative
    nz, ny, nx = 49, 49, 49
    z, y, x = np.meshgrid(np.linspace(0, 1, nz), np.linspace(0, 1, ny),
                          np.linspace(0, 1, nx), indexing="ij")
    u = conservative(x, y, z)
    f = np.zeros_like(u)
    o = oracle.compute_rhs(u, f, dt=1.0, threads=8)
    assert_tol(gpu_rhs(u, f, 1.0, strict=False), o)


_WS_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, {root!r})
import nasgen, oracle, paper_conf_icpp_tiankexc16_b200 as sr
sr.init(0)
for bench, cls in (("BT", "S"), ("SP", "W"), ("BT", "A"), ("BT", "C")):
    inp = nasgen.make_class(bench, cls, seed=1, B=1e-2)
    nz, ny, nx, _ = inp.u.shape
    c = sr.coeffs_nas(nx, ny, nz, inp.dt)
    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    o = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=8)
    for strict in (True, False):
        dr = torch.full_like(du, float("nan"))
        sr.rhs(du, df, dr, nx, c, strict=strict)
        torch.cuda.synchronize()
        g = sr.unpack(dr, nx)
        if strict:
            assert np.array_equal(g, o), (bench, cls)
        else:
            assert (np.abs(g - o) <= 1e-12 * np.abs(o) + 1e-14).all(), (bench, cls)
print("ws ok")
"""


def test_warp_specialised_kernel_parity():
    """The warp-specialised kernel (rhs_ws.cuh, SAFARA_WS=1: producer
    warpgroup computing rho_i/square into a shared-memory aux ring) is held to
    the same bar: STRICT bit-identical, production within c5 (own process:
    the knob is read once at init)."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", _WS_SCRIPT.format(root=root)],
                       env=dict(os.environ, SAFARA_WS="1"), capture_output=True, text=True,
                       timeout=600)
    assert r.returncode == 0 and "ws ok" in r.stdout, r.stderr[-2000:]


@pytest.mark.parametrize("cls,nchunks", [(("SP", "W"), 3), (("BT", "C"), 8)])
def test_host_e2e_unpadded_descriptor(cls, nchunks):
    """safara_rhs_host_ex on the unpadded NAS-native layout (sy = nx, the
    `dim` descriptor given explicitly): STRICT bit-identical to the oracle
    through host buffers, k-chunked copies and the kernel on sy = nx rows."""
    inp = nasgen.make_class(*cls, seed=8)
    nz, ny, nx, _ = inp.u.shape
    assert nx % 2 == 0

    def host(a):
        t = torch.empty((nz, 5, ny, nx), dtype=torch.float64).pin_memory()
        t.copy_(torch.from_numpy(np.ascontiguousarray(a)).permute(0, 3, 1, 2))
        return t

    hu, hf = host(inp.u), host(inp.forcing)
    hr = torch.zeros_like(hu).pin_memory()
    du, df, dr = (torch.empty(hu.shape, dtype=torch.float64, device="cuda") for _ in range(3))
    d = sr.Dims(nx, ny, nz, nx, ny * nx, 5 * ny * nx)
    c = sr.coeffs_nas(nx, ny, nz, inp.dt)
    sr.rhs_host_ex(hu, hf, hr, du, df, dr, d, c, strict=True, nchunks=nchunks)
    torch.cuda.synchronize()
    got = hr.permute(0, 2, 3, 1).numpy()
    assert np.array_equal(got, oracle_rhs(inp))


@pytest.mark.parametrize("cls,nchunks", [(("SP", "W"), 3), (("BT", "C"), 8)])
def test_host_e2e_pipelined_calls(cls, nchunks):
    """SAFARA_FLAG_PIPELINE: four back-to-back host calls on DIFFERENT inputs
    through the same device buffers, no synchronisation in between (the next
    call's H2D overlaps this call's last kernels and D2H): every call's rhs is
    still bit-identical (STRICT) to the oracle on its own inputs."""
    n = 4
    inps = [nasgen.make_class(*cls, seed=20 + s) for s in range(n)]
    nz, ny, nx, _ = inps[0].u.shape
    hus = [sr.pack(i.u, pin=True) for i in inps]
    hfs = [sr.pack(i.forcing, pin=True) for i in inps]
    hrs = [torch.zeros_like(hus[0]).pin_memory() for _ in range(n)]
    du, df, dr = (torch.empty(hus[0].shape, dtype=torch.float64, device="cuda") for _ in range(3))
    c = sr.coeffs_nas(nx, ny, nz, inps[0].dt)
    for s in range(n):
        sr.rhs_host(hus[s], hfs[s], hrs[s], du, df, dr, nx, c, strict=True, nchunks=nchunks,
                    pipeline=True)
    torch.cuda.synchronize()
    for s in range(n):
        assert np.array_equal(sr.unpack(hrs[s], nx), oracle_rhs(inps[s])), f"call {s}"

"""GPU parity of the 355.seismic dz loop (Fig. 8)
through the C ABI against the oracle: bit-identical (IEEE division, the
Fortran evaluation order), untouched points preserved, `dim`/`small` errors."""
import ctypes

import numpy as np
import pytest
import torch

import oracle
import paper_conf_icpp_tiankexc16_b200 as sr

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _init():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    sr.init(0)


def run(nx, ny, nz, seed, h=0.37):
    r = np.random.default_rng(seed)
    v = [r.standard_normal((nz, ny, nx)) for _ in range(3)]
    sy = sr.pitch(nx)

    def dev(a, fill=0.0):
        t = torch.full((nz, ny, sy), fill, dtype=torch.float64)
        t[..., :nx] = torch.from_numpy(a)
        return t.cuda()

    dv = [dev(a) for a in v]
    out = torch.full((nz, ny, sy), float("nan"), dtype=torch.float64, device="cuda")
    n0 = sr.launch_count()
    sr.seismic_dz(*dv, out, h, nx)
    torch.cuda.synchronize()
    assert sr.launch_count() == n0 + 1
    return out[..., :nx].cpu().numpy(), oracle.seismic_dz(*v, h)


@pytest.mark.parametrize("shape", [(12, 12, 12), (37, 9, 70), (162, 162, 162), (5, 3, 2),
                                   (33, 65, 17)])
def test_seismic_bitwise(shape):
    g, o = run(*shape, seed=sum(shape))
    assert np.array_equal(np.isnan(g), np.isnan(o)), "written ranges differ"
    assert np.array_equal(np.nan_to_num(g), np.nan_to_num(o))


def test_seismic_errors():
    L = sr._abi.lib()
    nz, ny, nx = 4, 4, 4
    t = [torch.zeros((nz, ny, 8), dtype=torch.float64, device="cuda") for _ in range(4)]
    p = [x.data_ptr() for x in t]
    d = sr.Dims3(nx, ny, nz, 8, 8 * ny)
    assert L.safara_seismic_dz(*p, ctypes.byref(d), 0.0, None) == -1           # h = 0
    assert L.safara_seismic_dz(p[0], p[1], p[2], p[0], ctypes.byref(d), 1.0, None) == -1
    bad = sr.Dims3(nx, ny, nz, 2, 8 * ny)
    assert L.safara_seismic_dz(*p, ctypes.byref(bad), 1.0, None) == -3          # sy < nx
    big = sr.Dims3(nx, ny, nz, 8, 1 << 30)
    assert L.safara_seismic_dz(*p, ctypes.byref(big), 1.0, None) == -5          # `small`
    assert L.safara_seismic_dz(*p, ctypes.byref(d), 1.0, None) == 0


@pytest.mark.parametrize("h", [0.37, 0.01, 1.0 / 3.0, 3.0, 1e-7, 12345.678, 2.0 ** -20, 0.7071067811865476])
def test_seismic_bitwise_wide_range(h):
    """Differences spanning +-250 binades and several spacings h: the division
    (IEEE x/h, or the library's correction form from RN(1/h)) must stay
    bit-identical to the oracle's IEEE division for every value."""
    nx, ny, nz = 67, 33, 41
    r = np.random.default_rng(int(h * 1e6) % 2**31)
    v = [r.standard_normal((nz, ny, nx)) * np.exp2(r.integers(-250, 250, (nz, ny, nx)))
         for _ in range(3)]
    sy = sr.pitch(nx)
    dv = []
    for a in v:
        t = torch.zeros((nz, ny, sy), dtype=torch.float64)
        t[..., :nx] = torch.from_numpy(a)
        dv.append(t.cuda())
    out = torch.full((nz, ny, sy), float("nan"), dtype=torch.float64, device="cuda")
    sr.seismic_dz(*dv, out, h, nx)
    g = out[..., :nx].cpu().numpy()
    o = oracle.seismic_dz(*v, h)
    assert np.array_equal(np.isnan(g), np.isnan(o))
    assert np.array_equal(np.nan_to_num(g), np.nan_to_num(o))


@pytest.mark.parametrize("h", [0.37, 1e-300, 1e300, -2.5])
def test_seismic_bitwise_special_values(h):
    """Signed zeros (-0 - +0 = -0), quotients at the subnormal / overflow edges
    and spacings h outside the range where the library forms x/h from RN(1/h):
    every value still equals the IEEE division bit for bit."""
    nx, ny, nz = 40, 9, 12
    r = np.random.default_rng(7)
    special = np.array([0.0, -0.0, 1e-310, -1e-310, 2.0 ** -1000, 1e300, -1e300, 5e-324,
                        1.7976931348623157e308, 1.0, -1.0, 3.0])
    v = [r.choice(special, size=(nz, ny, nx)) * r.choice([1.0, -1.0, 0.5], size=(nz, ny, nx))
         for _ in range(3)]
    sy = sr.pitch(nx)
    dv = []
    for a in v:
        t = torch.zeros((nz, ny, sy), dtype=torch.float64)
        t[..., :nx] = torch.from_numpy(a)
        dv.append(t.cuda())
    out = torch.full((nz, ny, sy), float("nan"), dtype=torch.float64, device="cuda")
    sr.seismic_dz(*dv, out, h, nx)
    g = out[..., :nx].cpu().numpy()
    with np.errstate(all="ignore"):
        o = oracle.seismic_dz(*v, h)
    written = ~np.isnan(o) | ~np.isnan(g)
    ok = (g.view(np.uint64) == o.view(np.uint64)) | (np.isnan(g) & np.isnan(o))
    assert ok[written].all()

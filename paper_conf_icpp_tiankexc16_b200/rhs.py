"""Torch-facing wrappers of the C ABI (argument marshalling only).

Canonical layout (include/safara.h): a field is a float64
tensor of shape ``(nz, 5, ny, sy)`` with ``sy = pitch(nx)``; element
(i, j, m, k) sits at offset ``i + sy*j + sm*m + sk*k``.  ``pack``/``unpack``
convert from/to the logical ``(nz, ny, nx, 5)`` layout used by ``nasgen`` and
the oracle; they are input/output marshalling, not part of the pass.
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

from ._abi import (SAFARA_AUX_BT, SAFARA_AUX_SP, SAFARA_FLAG_STRICT, SAFARA_FLAG_PIPELINE, SAFARA_IPC_HANDLE_BYTES,
                   SAFARA_PART_ALL, SAFARA_UNIQUE_ID_BYTES, BtCoeffs, Coeffs, Dims, Dims3,
                   KernelInfo, Peer, check, lib)

_initialised: set[int] = set()


def init(device: int | None = None) -> int:
    """safara_rhs_init for ``device`` (default: current CUDA device)."""
    if device is None:
        device = torch.cuda.current_device()
    if device not in _initialised:
        check(lib().safara_rhs_init(int(device)), "safara_rhs_init")
        _initialised.add(device)
    return device


def pitch(nx: int) -> int:
    return lib().safara_pitch(int(nx))


def canonical_dims(nx: int, ny: int, nz: int) -> Dims:
    d = Dims()
    check(lib().safara_dims_canonical(nx, ny, nz, ctypes.byref(d)), "safara_dims_canonical")
    return d


def validate_dims(d: Dims, nz_buf: int) -> int:
    return lib().safara_validate_dims(ctypes.byref(d), int(nz_buf))


def coeffs_nas(nx: int, ny: int, nz: int, dt: float) -> Coeffs:
    c = Coeffs()
    check(lib().safara_coeffs_nas(nx, ny, nz, float(dt), ctypes.byref(c)), "safara_coeffs_nas")
    return c


def empty_field(nx: int, ny: int, nplanes: int, device="cuda", pin: bool = False) -> torch.Tensor:
    """Uninitialised canonical field of ``nplanes`` k-planes."""
    t = torch.empty((nplanes, 5, ny, pitch(nx)), dtype=torch.float64,
                    device="cpu" if pin else device, pin_memory=pin)
    return t


def pack(a, device="cuda", pin: bool = False) -> torch.Tensor:
    """Logical (nz, ny, nx, 5) array -> canonical (nz, 5, ny, sy) tensor
    (pitch padding zero-filled)."""
    t = torch.as_tensor(np.ascontiguousarray(a) if isinstance(a, np.ndarray) else a,
                        dtype=torch.float64)
    nz, ny, nx, five = t.shape
    assert five == 5
    out = torch.zeros((nz, 5, ny, pitch(nx)), dtype=torch.float64,
                      device="cpu" if pin else device, pin_memory=pin)
    out[..., :nx] = t.permute(0, 3, 1, 2).to(out.device)
    return out


def unpack(t: torch.Tensor, nx: int) -> np.ndarray:
    """Canonical (nz, 5, ny, sy) tensor -> logical (nz, ny, nx, 5) numpy array."""
    return np.ascontiguousarray(t[..., :nx].permute(0, 2, 3, 1).cpu().numpy())


def _stream_ptr(stream) -> int | None:
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)


def _check_field(t: torch.Tensor, name: str):
    if t.dtype != torch.float64 or not t.is_cuda or not t.is_contiguous():
        raise ValueError(f"{name} must be a contiguous float64 CUDA tensor")


def _check_shape(t: torch.Tensor, shape: tuple, name: str):
    """The C side sizes its TMA maps and stores from the descriptor alone, so
    every tensor must really hold the planes the descriptor implies."""
    if tuple(t.shape) != tuple(shape):
        raise ValueError(f"{name} has shape {tuple(t.shape)}, expected {tuple(shape)}")


def _max_offset(d: Dims, nplanes: int, ncomp: int = 5) -> int:
    return (d.nx - 1) + d.sy * (d.ny - 1) + d.sm * (ncomp - 1) + d.sk * (nplanes - 1)


def _check_numel(t: torch.Tensor, d: Dims, nplanes: int, name: str):
    need = _max_offset(d, nplanes) + 1
    if t.numel() < need:
        raise ValueError(f"{name} holds {t.numel()} doubles, the descriptor reaches {need}")


def _canonical_fields(nx: int, fields, nplanes_u: int | None = None):
    """Check canonical (nplanes, 5, ny, pitch(nx)) tensors: fields[0] is u
    (nplanes_u planes if given, else the same as the others)."""
    ref = fields[1][0]
    nzl, five, ny, sy = ref.shape if ref.dim() == 4 else (None, None, None, None)
    if ref.dim() != 4 or five != 5 or sy != pitch(nx):
        raise ValueError(f"{fields[1][1]} must be canonical (nplanes, 5, ny, {pitch(nx)}), "
                         f"got {tuple(ref.shape)}")
    for i, (t, n) in enumerate(fields):
        want = (nplanes_u if (i == 0 and nplanes_u is not None) else nzl, 5, ny, sy)
        _check_shape(t, want, n)
    return nzl, ny


def rhs(u: torch.Tensor, forcing: torch.Tensor, out: torch.Tensor, nx: int, coeffs: Coeffs,
        strict: bool = False, stream=None, dims: Dims | None = None) -> torch.Tensor:
    """One compute_rhs pass: ``out <- F(u, forcing)`` on the GPU (async).

    Tensors are canonical ``(nz, 5, ny, sy)`` unless ``dims`` describes
    another stride order (then they are flat buffers of that layout).
    Canonical + production calls ``safara_rhs`` itself; STRICT or an explicit
    descriptor goes through ``safara_rhs_ex``."""
    for t, n in ((u, "u"), (forcing, "forcing"), (out, "out")):
        _check_field(t, n)
    if dims is None:
        nz, ny = _canonical_fields(nx, ((u, "u"), (forcing, "forcing"), (out, "out")))
        if not strict:
            # the north_star entry point itself: canonical layout, production
            check(lib().safara_rhs(u.data_ptr(), forcing.data_ptr(), out.data_ptr(), int(nx),
                                   int(ny), int(nz), ctypes.byref(coeffs), _stream_ptr(stream)),
                  "safara_rhs")
            return out
        dims = canonical_dims(nx, ny, nz)
    else:
        for t, n in ((u, "u"), (forcing, "forcing"), (out, "out")):
            _check_numel(t, dims, dims.nz, n)
    flags = SAFARA_FLAG_STRICT if strict else 0
    check(lib().safara_rhs_ex(u.data_ptr(), forcing.data_ptr(), out.data_ptr(),
                              ctypes.byref(dims), ctypes.byref(coeffs), flags,
                              _stream_ptr(stream)), "safara_rhs_ex")
    return out


def rhs_slab(u_slab: torch.Tensor, forcing_slab: torch.Tensor, out_slab: torch.Tensor,
             nx: int, nz: int, k0: int, coeffs: Coeffs, part: int = SAFARA_PART_ALL,
             strict: bool = False, stream=None) -> torch.Tensor:
    """z-slab pass: u_slab has nzl+4 planes (2 ghosts each side), forcing /
    out have nzl planes; this slab owns global planes [k0, k0+nzl)."""
    for t, n in ((u_slab, "u_slab"), (forcing_slab, "forcing_slab"), (out_slab, "out_slab")):
        _check_field(t, n)
    nzl = forcing_slab.shape[0]
    _, ny = _canonical_fields(nx, ((u_slab, "u_slab"), (forcing_slab, "forcing_slab"),
                                   (out_slab, "out_slab")), nplanes_u=nzl + 4)
    dims = canonical_dims(nx, ny, nz)
    flags = SAFARA_FLAG_STRICT if strict else 0
    check(lib().safara_rhs_slab(u_slab.data_ptr(), forcing_slab.data_ptr(), out_slab.data_ptr(),
                                ctypes.byref(dims), int(k0), int(nzl), ctypes.byref(coeffs),
                                flags, int(part), _stream_ptr(stream)), "safara_rhs_slab")
    return out_slab


def rhs_peer(u_slab: torch.Tensor, forcing_slab: torch.Tensor, out_slab: torch.Tensor,
             nx: int, nz: int, k0: int, peer: Peer, coeffs: Coeffs, strict: bool = False,
             stream=None) -> torch.Tensor:
    """f2: z-slab pass whose halo planes are read from the neighbours' u slabs
    through the peer pointers in ``peer`` (safara_peer_t); one launch, no
    exchange.  Slab tensors as in :func:`rhs_slab` (ghost planes unused)."""
    for t, n in ((u_slab, "u_slab"), (forcing_slab, "forcing_slab"), (out_slab, "out_slab")):
        _check_field(t, n)
    nzl = forcing_slab.shape[0]
    _, ny = _canonical_fields(nx, ((u_slab, "u_slab"), (forcing_slab, "forcing_slab"),
                                   (out_slab, "out_slab")), nplanes_u=nzl + 4)
    dims = canonical_dims(nx, ny, nz)
    flags = SAFARA_FLAG_STRICT if strict else 0
    check(lib().safara_rhs_peer(u_slab.data_ptr(), forcing_slab.data_ptr(), out_slab.data_ptr(),
                                ctypes.byref(dims), int(k0), int(nzl), ctypes.byref(peer),
                                ctypes.byref(coeffs), flags, _stream_ptr(stream)),
          "safara_rhs_peer")
    return out_slab


# ---- the sharded pass, library-owned NCCL communicator ----

def get_unique_id() -> bytes:
    """safara_get_unique_id: SAFARA_UNIQUE_ID_BYTES opaque bytes (rank 0)."""
    b = ctypes.create_string_buffer(SAFARA_UNIQUE_ID_BYTES)
    check(lib().safara_get_unique_id(b), "safara_get_unique_id")
    return b.raw


def shard_init(uid: bytes, rank: int, nranks: int, device: int) -> int:
    """safara_shard_init; returns the opaque shard handle (an address)."""
    if len(uid) != SAFARA_UNIQUE_ID_BYTES:
        raise ValueError(f"unique id must be {SAFARA_UNIQUE_ID_BYTES} bytes")
    h = ctypes.c_void_p()
    check(lib().safara_shard_init(uid, int(rank), int(nranks), int(device), ctypes.byref(h)),
          "safara_shard_init")
    return int(h.value)


def shard_finalize(handle: int) -> None:
    check(lib().safara_shard_finalize(handle), "safara_shard_finalize")


def shard_rank(handle: int) -> tuple[int, int]:
    r, n = ctypes.c_int(), ctypes.c_int()
    check(lib().safara_shard_rank(handle, ctypes.byref(r), ctypes.byref(n)), "safara_shard_rank")
    return r.value, n.value


def rhs_sharded(handle: int, u_slab: torch.Tensor, forcing_slab: torch.Tensor,
                out_slab: torch.Tensor, nx: int, nz: int, k0: int, coeffs: Coeffs,
                strict: bool = False, stream=None) -> torch.Tensor:
    """safara_rhs_sharded(_ex): NCCL halo exchange into u_slab's ghost planes
    overlapped with the interior planes, then the edge planes (async)."""
    for t, n in ((u_slab, "u_slab"), (forcing_slab, "forcing_slab"), (out_slab, "out_slab")):
        _check_field(t, n)
    nzl = forcing_slab.shape[0]
    _, ny = _canonical_fields(nx, ((u_slab, "u_slab"), (forcing_slab, "forcing_slab"),
                                   (out_slab, "out_slab")), nplanes_u=nzl + 4)
    L = lib()
    if strict:
        dims = canonical_dims(nx, ny, nz)
        rc = L.safara_rhs_sharded_ex(handle, u_slab.data_ptr(), forcing_slab.data_ptr(),
                                     out_slab.data_ptr(), ctypes.byref(dims), int(k0), int(nzl),
                                     ctypes.byref(coeffs), SAFARA_FLAG_STRICT, _stream_ptr(stream))
        check(rc, "safara_rhs_sharded_ex")
    else:
        rc = L.safara_rhs_sharded(handle, u_slab.data_ptr(), forcing_slab.data_ptr(),
                                  out_slab.data_ptr(), int(nx), int(ny), int(nz), int(k0),
                                  int(nzl), ctypes.byref(coeffs), _stream_ptr(stream))
        check(rc, "safara_rhs_sharded")
    return out_slab


def shard_rms(handle: int, r_slab: torch.Tensor, nx: int, nz: int, k0: int, stream=None,
              out: torch.Tensor | None = None) -> torch.Tensor:
    """safara_shard_rms: NPB rhs_norm over every rank's slab (NCCL all-reduce
    of the per-slab sums, finished on the device); 5 device doubles (async)."""
    _check_field(r_slab, "rhs_slab")
    nzl, ny = _canonical_fields(nx, ((r_slab, "rhs_slab"), (r_slab, "rhs_slab")))
    dims = canonical_dims(nx, ny, nz)
    work = _work_for(r_slab, stream)
    if out is None:
        out = torch.empty(5, dtype=torch.float64, device=r_slab.device)
    check(lib().safara_shard_rms(handle, r_slab.data_ptr(), ctypes.byref(dims), int(k0), int(nzl),
                                 work.data_ptr(), out.data_ptr(), _stream_ptr(stream)),
          "safara_shard_rms")
    return out


def ipc_get(t: torch.Tensor) -> tuple[bytes, int]:
    """(handle bytes, offset) exporting the allocation that holds ``t``."""
    h = ctypes.create_string_buffer(SAFARA_IPC_HANDLE_BYTES)
    off = ctypes.c_int64()
    check(lib().safara_ipc_get(t.data_ptr(), h, ctypes.byref(off)), "safara_ipc_get")
    return h.raw, int(off.value)


def ipc_open(handle: bytes, offset: int) -> int:
    """Map another process's export on the current device; returns the pointer."""
    p = ctypes.c_void_p()
    check(lib().safara_ipc_open(handle, int(offset), ctypes.byref(p)), "safara_ipc_open")
    return int(p.value)


def ipc_close(ptr: int, offset: int) -> None:
    check(lib().safara_ipc_close(ptr, int(offset)), "safara_ipc_close")


def rhs_host(u_host: torch.Tensor, f_host: torch.Tensor, r_host: torch.Tensor,
             u_dev: torch.Tensor, f_dev: torch.Tensor, r_dev: torch.Tensor, nx: int,
             coeffs: Coeffs, strict: bool = False, nchunks: int = 8, stream=None,
             pipeline: bool = False):
    """End-to-end pass on host (pinned) canonical tensors through device buffers
    (pipeline: SAFARA_FLAG_PIPELINE, see include/safara.h)."""
    nz, ny = _canonical_fields(nx, ((u_host, "u_host"), (f_host, "f_host"), (r_host, "r_host")))
    for t, n in ((u_dev, "u_dev"), (f_dev, "f_dev"), (r_dev, "r_dev")):
        _check_field(t, n)
        _check_shape(t, tuple(u_host.shape), n)
    flags = (SAFARA_FLAG_STRICT if strict else 0) | (SAFARA_FLAG_PIPELINE if pipeline else 0)
    check(lib().safara_rhs_host(u_host.data_ptr(), f_host.data_ptr(), r_host.data_ptr(),
                                u_dev.data_ptr(), f_dev.data_ptr(), r_dev.data_ptr(),
                                nx, ny, nz, ctypes.byref(coeffs), flags, int(nchunks),
                                _stream_ptr(stream)), "safara_rhs_host")
    return r_host


def rhs_host_ex(u_host: torch.Tensor, f_host: torch.Tensor, r_host: torch.Tensor,
                u_dev: torch.Tensor, f_dev: torch.Tensor, r_dev: torch.Tensor, dims: Dims,
                coeffs: Coeffs, strict: bool = False, nchunks: int = 8, stream=None,
                pipeline: bool = False):
    """End-to-end pass on host (pinned) arrays in the layout `dims` describes
    (e.g. the unpadded sy = nx layout) through device buffers of the same layout."""
    need = (_max_offset(dims, dims.nz) + 1)
    for t, n in ((u_host, "u_host"), (f_host, "f_host"), (r_host, "r_host")):
        if t.dtype != torch.float64 or not t.is_contiguous() or t.device.type != "cpu":
            raise ValueError(f"{n}: contiguous float64 CPU tensor expected")
        if t.numel() < need:
            raise ValueError(f"{n}: {t.numel()} elements < the descriptor's {need}")
    for t, n in ((u_dev, "u_dev"), (f_dev, "f_dev"), (r_dev, "r_dev")):
        _check_field(t, n)
        if t.numel() < need:
            raise ValueError(f"{n}: {t.numel()} elements < the descriptor's {need}")
    flags = (SAFARA_FLAG_STRICT if strict else 0) | (SAFARA_FLAG_PIPELINE if pipeline else 0)
    check(lib().safara_rhs_host_ex(u_host.data_ptr(), f_host.data_ptr(), r_host.data_ptr(),
                                   u_dev.data_ptr(), f_dev.data_ptr(), r_dev.data_ptr(),
                                   ctypes.byref(dims), ctypes.byref(coeffs), flags, int(nchunks),
                                   _stream_ptr(stream)), "safara_rhs_host_ex")
    return r_host


def launch_count() -> int:
    return int(lib().safara_launch_count())


def kernel_info(strict: bool = False) -> dict:
    k = KernelInfo()
    check(lib().safara_kernel_info(1 if strict else 0, ctypes.byref(k)), "safara_kernel_info")
    return {f: getattr(k, f) for f, _ in KernelInfo._fields_}


# ---- step-0 auxiliary fields and the rhs norm -------------

AUX_NAMES = ("rho_i", "us", "vs", "ws", "square", "qs", "speed")


def empty_aux(nx: int, ny: int, nplanes: int, naux: int = SAFARA_AUX_BT,
              device="cuda") -> torch.Tensor:
    """Canonical aux array (nplanes, naux, ny, sy): component c of (i, j, p)
    at i + sy*j + sm*c + naux*sm*p (include/safara.h)."""
    return torch.empty((nplanes, naux, ny, pitch(nx)), dtype=torch.float64, device=device)


def unpack_aux(t: torch.Tensor, nx: int) -> np.ndarray:
    """Canonical (nz, naux, ny, sy) -> logical (nz, ny, nx, naux)."""
    return np.ascontiguousarray(t[..., :nx].permute(0, 2, 3, 1).cpu().numpy())


def rhs_aux(u: torch.Tensor, forcing: torch.Tensor, out: torch.Tensor, aux: torch.Tensor,
            nx: int, coeffs: Coeffs, strict: bool = False, stream=None,
            dims: Dims | None = None) -> torch.Tensor:
    """compute_rhs pass that also writes the step-0 fields into ``aux``
    (naux = aux.shape[1] for canonical tensors: 6 BT or 7 with SP speed)."""
    for t, n in ((u, "u"), (forcing, "forcing"), (out, "out"), (aux, "aux")):
        _check_field(t, n)
    if dims is None:
        nz, ny = _canonical_fields(nx, ((u, "u"), (forcing, "forcing"), (out, "out")))
        dims = canonical_dims(nx, ny, nz)
        if aux.dim() != 4 or aux.shape[1] not in (SAFARA_AUX_BT, SAFARA_AUX_SP):
            raise ValueError(f"aux must be (nz, 6|7, ny, sy), got {tuple(aux.shape)}")
        _check_shape(aux, (nz, aux.shape[1], ny, pitch(nx)), "aux")
    else:
        for t, n in ((u, "u"), (forcing, "forcing"), (out, "out")):
            _check_numel(t, dims, dims.nz, n)
    naux = int(aux.shape[1]) if aux.dim() == 4 else SAFARA_AUX_BT
    flags = SAFARA_FLAG_STRICT if strict else 0
    check(lib().safara_rhs_aux(u.data_ptr(), forcing.data_ptr(), out.data_ptr(), aux.data_ptr(),
                               naux, ctypes.byref(dims), ctypes.byref(coeffs), flags,
                               _stream_ptr(stream)), "safara_rhs_aux")
    return aux


def rhs_slab_aux(u_slab, forcing_slab, out_slab, aux_slab, nx: int, nz: int, k0: int,
                 coeffs: Coeffs, part: int = SAFARA_PART_ALL, strict: bool = False,
                 stream=None) -> torch.Tensor:
    for t, n in ((u_slab, "u_slab"), (forcing_slab, "forcing_slab"), (out_slab, "out_slab"),
                 (aux_slab, "aux_slab")):
        _check_field(t, n)
    nzl = forcing_slab.shape[0]
    _, ny = _canonical_fields(nx, ((u_slab, "u_slab"), (forcing_slab, "forcing_slab"),
                                   (out_slab, "out_slab")), nplanes_u=nzl + 4)
    if aux_slab.dim() != 4 or aux_slab.shape[1] not in (SAFARA_AUX_BT, SAFARA_AUX_SP):
        raise ValueError(f"aux_slab must be (nzl, 6|7, ny, sy), got {tuple(aux_slab.shape)}")
    _check_shape(aux_slab, (nzl, aux_slab.shape[1], ny, pitch(nx)), "aux_slab")
    dims = canonical_dims(nx, ny, nz)
    flags = SAFARA_FLAG_STRICT if strict else 0
    check(lib().safara_rhs_slab_aux(u_slab.data_ptr(), forcing_slab.data_ptr(),
                                    out_slab.data_ptr(), aux_slab.data_ptr(),
                                    int(aux_slab.shape[1]), ctypes.byref(dims), int(k0), int(nzl),
                                    ctypes.byref(coeffs), flags, int(part), _stream_ptr(stream)),
          "safara_rhs_slab_aux")
    return aux_slab


# scratch of safara_norm_work_doubles() doubles, one per (device, stream): two
# reductions on different streams never share partials
_norm_work: dict[tuple[int, int], torch.Tensor] = {}


def _work_for(r: torch.Tensor, stream) -> torch.Tensor:
    dev = r.device.index if r.device.index is not None else torch.cuda.current_device()
    key = (dev, int(_stream_ptr(stream) or 0))
    work = _norm_work.get(key)
    if work is None:
        work = torch.empty(lib().safara_norm_work_doubles(), dtype=torch.float64, device=r.device)
        _norm_work[key] = work
    return work


# safara_rhs_fused scratch: norm work + 8 words, word 0 a CTA counter that
# must start at zero (zeros at allocation; the library leaves it zero)
_fused_work: dict[tuple[int, int], torch.Tensor] = {}


def _fused_work_for(r: torch.Tensor, stream) -> torch.Tensor:
    dev = r.device.index if r.device.index is not None else torch.cuda.current_device()
    key = (dev, int(_stream_ptr(stream) or 0))
    work = _fused_work.get(key)
    if work is None:
        work = torch.zeros(lib().safara_norm_work_doubles() + 8, dtype=torch.float64,
                           device=r.device)
        _fused_work[key] = work
    return work


def rhs_sumsq(r: torch.Tensor, nx: int, nz: int | None = None, k0: int = 0, stream=None,
              out: torch.Tensor | None = None, dims: Dims | None = None) -> torch.Tensor:
    """Per-component sums of rhs^2 over the interior points of the planes
    ``r`` holds (plane p = global k0+p); a 5-element device tensor (async)."""
    _check_field(r, "rhs")
    nzl = r.shape[0]
    nz = nzl if nz is None else nz
    if dims is None:
        _, ny = _canonical_fields(nx, ((r, "rhs"), (r, "rhs")))
        dims = canonical_dims(nx, ny, nz)
    else:
        _check_numel(r, dims, nzl, "rhs")
    work = _work_for(r, stream)
    if out is None:
        out = torch.empty(5, dtype=torch.float64, device=r.device)
    check(lib().safara_rhs_sumsq(r.data_ptr(), ctypes.byref(dims), int(k0), int(nzl),
                                 work.data_ptr(), out.data_ptr(), _stream_ptr(stream)),
          "safara_rhs_sumsq")
    return out


def rhs_rms(r: torch.Tensor, nx: int, stream=None, out: torch.Tensor | None = None) -> torch.Tensor:
    """NPB rhs_norm of a full-grid canonical rhs, computed entirely on the
    device (safara_rhs_rms): a 5-element device tensor sqrt(sum rhs(m)^2 /
    ((nx-2)(ny-2)(nz-2))) (async)."""
    _check_field(r, "rhs")
    nz, ny = _canonical_fields(nx, ((r, "rhs"), (r, "rhs")))
    dims = canonical_dims(nx, ny, nz)
    work = _work_for(r, stream)
    if out is None:
        out = torch.empty(5, dtype=torch.float64, device=r.device)
    check(lib().safara_rhs_rms(r.data_ptr(), ctypes.byref(dims), work.data_ptr(), out.data_ptr(),
                               _stream_ptr(stream)), "safara_rhs_rms")
    return out


def rhs_fused(u: torch.Tensor, forcing: torch.Tensor, out: torch.Tensor, nx: int,
              coeffs: Coeffs, aux: torch.Tensor | None = None, rms: bool | torch.Tensor = True,
              strict: bool = False, stream=None) -> torch.Tensor | None:
    """safara_rhs_fused: one pass writing rhs, optionally the aux fields, and
    (rms=True or a 5-element device tensor) NPB rhs_norm accumulated in the
    store epilogue.  Returns the rms tensor (or None)."""
    for t, n in ((u, "u"), (forcing, "forcing"), (out, "out")):
        _check_field(t, n)
    nz, ny = _canonical_fields(nx, ((u, "u"), (forcing, "forcing"), (out, "out")))
    dims = canonical_dims(nx, ny, nz)
    naux = 0
    if aux is not None:
        _check_field(aux, "aux")
        if aux.dim() != 4 or aux.shape[1] not in (SAFARA_AUX_BT, SAFARA_AUX_SP):
            raise ValueError(f"aux must be (nz, 6|7, ny, sy), got {tuple(aux.shape)}")
        _check_shape(aux, (nz, aux.shape[1], ny, pitch(nx)), "aux")
        naux = int(aux.shape[1])
    out_rms = None
    if rms is not False and rms is not None:
        out_rms = rms if isinstance(rms, torch.Tensor) else torch.empty(
            5, dtype=torch.float64, device=u.device)
    work = _fused_work_for(u, stream) if out_rms is not None else None
    check(lib().safara_rhs_fused(u.data_ptr(), forcing.data_ptr(), out.data_ptr(),
                                 aux.data_ptr() if aux is not None else None, naux,
                                 work.data_ptr() if work is not None else None,
                                 out_rms.data_ptr() if out_rms is not None else None,
                                 ctypes.byref(dims), ctypes.byref(coeffs),
                                 SAFARA_FLAG_STRICT if strict else 0, _stream_ptr(stream)),
          "safara_rhs_fused")
    return out_rms


def rhs_norm(r: torch.Tensor, nx: int, stream=None) -> np.ndarray:
    """NPB rhs_norm of a full-grid canonical rhs as a host numpy array
    (safara_rhs_rms, then a device->host copy: synchronises)."""
    return rhs_rms(r, nx, stream=stream).cpu().numpy()


# ---- the 355.seismic dz loop (Fig. 8) --------

def seismic_dz(vz1: torch.Tensor, vz2: torch.Tensor, vz3: torch.Tensor, out: torch.Tensor,
               h: float, nx: int, stream=None) -> torch.Tensor:
    """value_dz of Fig. 8 into ``out`` for (nz, ny, sy) float64 CUDA tensors
    sharing one pitched layout (sy >= nx): j in [1, ny-1], i in [0, nx-2],
    k in [1, nz-1]; other points untouched."""
    for t, n in ((vz1, "vz1"), (vz2, "vz2"), (vz3, "vz3"), (out, "value_dz")):
        _check_field(t, n)
        if t.shape != vz1.shape or t.dim() != 3:
            raise ValueError("vz1, vz2, vz3 and value_dz must share one (nz, ny, sy) shape")
    nz, ny, sy = vz1.shape
    d = Dims3(nx, ny, nz, sy, sy * ny)
    check(lib().safara_seismic_dz(vz1.data_ptr(), vz2.data_ptr(), vz3.data_ptr(), out.data_ptr(),
                                  ctypes.byref(d), float(h), _stream_ptr(stream)),
          "safara_seismic_dz")
    return out


# ---- a whole NPB BT time step ---------------------------

def bt_coeffs_nas(nx: int, ny: int, nz: int, dt: float) -> BtCoeffs:
    c = BtCoeffs()
    check(lib().safara_bt_coeffs_nas(nx, ny, nz, float(dt), ctypes.byref(c)),
          "safara_bt_coeffs_nas")
    return c


class BtState:
    """Device state of an NPB BT run on canonical tensors: u (updated in
    place), forcing, and the rhs / aux / solver scratch the step overwrites."""

    def __init__(self, u: torch.Tensor, forcing: torch.Tensor, nx: int, dt: float):
        _check_field(u, "u")
        _check_field(forcing, "forcing")
        nz, ny = _canonical_fields(nx, ((u, "u"), (forcing, "forcing"), (forcing, "forcing")))
        self.nx, self.ny, self.nz, self.dt = nx, ny, nz, dt
        self.u, self.forcing = u, forcing
        self.rhs = torch.empty_like(u)
        self.aux = torch.empty((nz, SAFARA_AUX_BT, ny, pitch(nx)), dtype=torch.float64,
                               device=u.device)
        w = lib().safara_bt_work_doubles(nx, ny, nz)
        check(min(w, 0), "safara_bt_work_doubles")
        self.work = torch.empty(w, dtype=torch.float64, device=u.device)
        self.dims = canonical_dims(nx, ny, nz)
        self.coeffs = coeffs_nas(nx, ny, nz, dt)
        self.bt = bt_coeffs_nas(nx, ny, nz, dt)

    def step(self, strict: bool = False, stream=None):
        """One ADI step: safara_bt_step (rhs_aux, x/y/z_solve, add; 5 launches)."""
        check(lib().safara_bt_step(self.u.data_ptr(), self.forcing.data_ptr(),
                                   self.rhs.data_ptr(), self.aux.data_ptr(), self.work.data_ptr(),
                                   ctypes.byref(self.dims), ctypes.byref(self.coeffs),
                                   ctypes.byref(self.bt), SAFARA_FLAG_STRICT if strict else 0,
                                   _stream_ptr(stream)), "safara_bt_step")

    def solve(self, direction: int, stream=None):
        """One line solve of self.rhs in place (aux must hold u's fields)."""
        check(lib().safara_bt_solve(int(direction), self.u.data_ptr(), self.aux.data_ptr(),
                                    self.rhs.data_ptr(), self.work.data_ptr(),
                                    ctypes.byref(self.dims), ctypes.byref(self.bt),
                                    _stream_ptr(stream)), "safara_bt_solve")

    def verify_norms(self, u_exact: torch.Tensor, strict: bool = False, stream=None):
        """NPB BT verify on the device: (xce, xcr) as 5-element device tensors,
        xce = error_norm(u, u_exact), xcr = rhs_norm(compute_rhs(u)) / dt."""
        _check_shape(u_exact, tuple(self.u.shape), "u_exact")
        work = _work_for(self.u, stream)
        xce = torch.empty(5, dtype=torch.float64, device=self.u.device)
        check(lib().safara_error_norm(self.u.data_ptr(), u_exact.data_ptr(),
                                      ctypes.byref(self.dims), work.data_ptr(), xce.data_ptr(),
                                      _stream_ptr(stream)), "safara_error_norm")
        rhs(self.u, self.forcing, self.rhs, self.nx, self.coeffs, strict=strict, stream=stream)
        xcr = rhs_rms(self.rhs, self.nx, stream=stream)
        return xce, xcr / self.dt

"""ctypes declarations of the C ABI in include/safara.h (argument marshalling only).

Loading fails loudly if the in-tree ``libsafara_rhs.so`` is missing: there is
no CPU or PyTorch fallback for any step of the pass.
"""
from __future__ import annotations

import ctypes
import os
import re
import threading

PKG = os.path.dirname(os.path.abspath(__file__))
# SAFARA_LIB overrides the library path (A/B experiments with variant builds).
LIB_PATH = os.environ.get("SAFARA_LIB") or os.path.join(PKG, "libsafara_rhs.so")
HEADER = os.path.join(os.path.dirname(PKG), "include", "safara.h")

SAFARA_OK = 0
SAFARA_FLAG_STRICT = 0x1
SAFARA_FLAG_PIPELINE = 0x2
SAFARA_PART_ALL, SAFARA_PART_INTERIOR, SAFARA_PART_EDGE = 0, 1, 2
SAFARA_AUX_BT, SAFARA_AUX_SP = 6, 7


class SafaraError(RuntimeError):
    def __init__(self, code: int, where: str):
        self.code = code
        super().__init__(f"{where}: {strerror(code)} (code {code})")


class Dims(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in ("nx", "ny", "nz", "sy", "sm", "sk")]


class Coeffs(ctypes.Structure):
    _fields_ = [(n, ctypes.c_double) for n in
                ("dt", "dssp", "c1", "c2", "con43", "tx2", "ty2", "tz2")] + [
        (n, ctypes.c_double * 5) for n in ("dxt", "dyt", "dzt", "xxcon", "yycon", "zzcon")]


class BtCoeffs(ctypes.Structure):
    """safara_bt_coeffs_t."""
    _fields_ = [(n, ctypes.c_double) for n in
                ("dt", "c1", "c2", "c3c4", "c1c5", "con43", "tx1", "tx2", "ty1", "ty2", "tz1",
                 "tz2")] + [(n, ctypes.c_double * 5) for n in ("dx", "dy", "dz")]


class Dims3(ctypes.Structure):
    """safara_dims3_t: the shared 3-D descriptor of the seismic dz loop."""
    _fields_ = [(n, ctypes.c_int32) for n in ("nx", "ny", "nz", "sy", "sk")]


class KernelInfo(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int) for n in
                ("regs_per_thread", "local_bytes", "smem_bytes", "threads_per_cta",
                 "ctas_per_sm", "tile_x", "tile_y", "stages")]


class Peer(ctypes.Structure):
    """safara_peer_t."""
    _fields_ = [("u_lo", ctypes.c_void_p), ("u_hi", ctypes.c_void_p),
                ("k0_lo", ctypes.c_int32), ("k0_hi", ctypes.c_int32),
                ("flags", ctypes.c_void_p), ("flags_lo", ctypes.c_void_p),
                ("flags_hi", ctypes.c_void_p), ("epoch", ctypes.c_uint64)]


SAFARA_PEER_WORDS = 8
SAFARA_PEER_LO_READY, SAFARA_PEER_HI_READY, SAFARA_PEER_LO_DONE, SAFARA_PEER_HI_DONE = 0, 1, 2, 3
SAFARA_PEER_ARRIVED, SAFARA_PEER_TIMEOUTS = 4, 5
SAFARA_PEER_TIMEOUT_WORDS, SAFARA_PEER_EPOCH_WORD = 6, 7
SAFARA_PEER_EPOCH_AUTO = 0xFFFFFFFFFFFFFFFF
SAFARA_IPC_HANDLE_BYTES = 64
SAFARA_UNIQUE_ID_BYTES = 128
SAFARA_ERR_NCCL = -9

_lock = threading.Lock()
_lib = None

_dp = ctypes.c_void_p  # device / host pointers travel as plain addresses
_SIGS = {
    "safara_coeffs_nas": ([ctypes.c_int] * 3 + [ctypes.c_double, ctypes.POINTER(Coeffs)], ctypes.c_int),
    "safara_rhs_init": ([ctypes.c_int], ctypes.c_int),
    "safara_pitch": ([ctypes.c_int], ctypes.c_int),
    "safara_dims_canonical": ([ctypes.c_int] * 3 + [ctypes.POINTER(Dims)], ctypes.c_int),
    "safara_validate_dims": ([ctypes.POINTER(Dims), ctypes.c_int], ctypes.c_int),
    "safara_rhs": ([_dp, _dp, _dp] + [ctypes.c_int] * 3 + [ctypes.POINTER(Coeffs), _dp], ctypes.c_int),
    "safara_rhs_ex": ([_dp, _dp, _dp, ctypes.POINTER(Dims), ctypes.POINTER(Coeffs), ctypes.c_int, _dp],
                      ctypes.c_int),
    "safara_rhs_slab": ([_dp, _dp, _dp, ctypes.POINTER(Dims), ctypes.c_int, ctypes.c_int,
                         ctypes.POINTER(Coeffs), ctypes.c_int, ctypes.c_int, _dp], ctypes.c_int),
    "safara_rhs_host": ([_dp] * 6 + [ctypes.c_int] * 3 + [ctypes.POINTER(Coeffs), ctypes.c_int,
                                                           ctypes.c_int, _dp], ctypes.c_int),
    "safara_rhs_host_ex": ([_dp] * 6 + [ctypes.POINTER(Dims), ctypes.POINTER(Coeffs), ctypes.c_int,
                            ctypes.c_int, _dp], ctypes.c_int),
    "safara_rhs_aux": ([_dp, _dp, _dp, _dp, ctypes.c_int, ctypes.POINTER(Dims),
                        ctypes.POINTER(Coeffs), ctypes.c_int, _dp], ctypes.c_int),
    "safara_rhs_slab_aux": ([_dp, _dp, _dp, _dp, ctypes.c_int, ctypes.POINTER(Dims), ctypes.c_int,
                             ctypes.c_int, ctypes.POINTER(Coeffs), ctypes.c_int, ctypes.c_int, _dp],
                            ctypes.c_int),
    "safara_rhs_peer": ([_dp, _dp, _dp, ctypes.POINTER(Dims), ctypes.c_int, ctypes.c_int,
                         ctypes.POINTER(Peer), ctypes.POINTER(Coeffs), ctypes.c_int, _dp],
                        ctypes.c_int),
    "safara_ipc_get": ([_dp, ctypes.c_char_p, ctypes.POINTER(ctypes.c_int64)], ctypes.c_int),
    "safara_ipc_open": ([ctypes.c_char_p, ctypes.c_int64, ctypes.POINTER(ctypes.c_void_p)],
                        ctypes.c_int),
    "safara_ipc_close": ([_dp, ctypes.c_int64], ctypes.c_int),
    "safara_norm_work_doubles": ([], ctypes.c_int),
    "safara_rhs_sumsq": ([_dp, ctypes.POINTER(Dims), ctypes.c_int, ctypes.c_int, _dp, _dp, _dp],
                         ctypes.c_int),
    "safara_seismic_dz": ([_dp] * 4 + [ctypes.POINTER(Dims3), ctypes.c_double, _dp], ctypes.c_int),
    "safara_rhs_rms": ([_dp, ctypes.POINTER(Dims), _dp, _dp, _dp], ctypes.c_int),
    "safara_rhs_fused": ([_dp, _dp, _dp, _dp, ctypes.c_int, _dp, _dp, ctypes.POINTER(Dims),
                          ctypes.POINTER(Coeffs), ctypes.c_int, _dp], ctypes.c_int),
    "safara_get_unique_id": ([ctypes.c_char_p], ctypes.c_int),
    "safara_shard_init": ([ctypes.c_char_p, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                           ctypes.POINTER(ctypes.c_void_p)], ctypes.c_int),
    "safara_rhs_sharded": ([_dp, _dp, _dp, _dp] + [ctypes.c_int] * 5 + [ctypes.POINTER(Coeffs), _dp],
                           ctypes.c_int),
    "safara_rhs_sharded_ex": ([_dp, _dp, _dp, _dp, ctypes.POINTER(Dims), ctypes.c_int, ctypes.c_int,
                              ctypes.POINTER(Coeffs), ctypes.c_int, _dp], ctypes.c_int),
    "safara_shard_rms": ([_dp, _dp, ctypes.POINTER(Dims), ctypes.c_int, ctypes.c_int, _dp, _dp, _dp],
                         ctypes.c_int),
    "safara_shard_rank": ([_dp, ctypes.POINTER(ctypes.c_int), ctypes.POINTER(ctypes.c_int)],
                          ctypes.c_int),
    "safara_shard_finalize": ([_dp], ctypes.c_int),
    "safara_bt_coeffs_nas": ([ctypes.c_int] * 3 + [ctypes.c_double, ctypes.POINTER(BtCoeffs)],
                             ctypes.c_int),
    "safara_bt_work_doubles": ([ctypes.c_int] * 3, ctypes.c_int),
    "safara_bt_solve": ([ctypes.c_int, _dp, _dp, _dp, _dp, ctypes.POINTER(Dims),
                         ctypes.POINTER(BtCoeffs), _dp], ctypes.c_int),
    "safara_bt_add": ([_dp, _dp, ctypes.POINTER(Dims), _dp], ctypes.c_int),
    "safara_bt_step": ([_dp] * 5 + [ctypes.POINTER(Dims), ctypes.POINTER(Coeffs),
                                    ctypes.POINTER(BtCoeffs), ctypes.c_int, _dp], ctypes.c_int),
    "safara_error_norm": ([_dp, _dp, ctypes.POINTER(Dims), _dp, _dp, _dp], ctypes.c_int),
    "safara_launch_count": ([], ctypes.c_int64),
    "safara_kernel_info": ([ctypes.c_int, ctypes.POINTER(KernelInfo)], ctypes.c_int),
    "safara_strerror": ([ctypes.c_int], ctypes.c_char_p),
}


def header_symbols() -> list[str]:
    """Function names declared in include/safara.h."""
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"\b(safara_[a-z_0-9]+)\s*\(", txt)))


def lib():
    """The loaded library (raises if it was not built)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise RuntimeError(
                    f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; "
                    "g.build()'` (no fallback exists)")
            L = ctypes.CDLL(LIB_PATH)
            for name, (args, res) in _SIGS.items():
                if os.environ.get("SAFARA_LIB") and not hasattr(L, name):
                    continue  # A/B builds of older revisions may predate an entry point
                fn = getattr(L, name)
                fn.argtypes = args
                fn.restype = res
            _lib = L
    return _lib


def strerror(code: int) -> str:
    return lib().safara_strerror(int(code)).decode()


def check(code: int, where: str) -> None:
    if code != SAFARA_OK:
        raise SafaraError(code, where)

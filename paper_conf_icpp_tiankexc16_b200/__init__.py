"""B200-native (sm_100a) NAS BT/SP ``compute_rhs`` -- thin Python binding.

The computation lives in ``libsafara_rhs.so`` (C ABI: include/safara.h);
this package only marshals torch tensors into that ABI.  PyTorch supplies
device memory, streams and process groups.  See DESIGN.md.
"""
from ._abi import (SAFARA_AUX_BT, SAFARA_AUX_SP, SAFARA_FLAG_STRICT, SAFARA_PART_ALL,
                   SAFARA_PART_EDGE, SAFARA_PART_INTERIOR, Coeffs, Dims, Dims3, Peer, SafaraError)
from ._abi import strerror
from .rhs import (AUX_NAMES, BtState, bt_coeffs_nas, canonical_dims, coeffs_nas, empty_aux, empty_field,
                  get_unique_id, init, ipc_close, ipc_get, ipc_open, kernel_info, launch_count,
                  pack, pitch, rhs, rhs_aux, rhs_fused, rhs_host, rhs_host_ex, rhs_norm, rhs_peer, rhs_rms, rhs_sharded,
                  rhs_slab, rhs_slab_aux, rhs_sumsq, seismic_dz, shard_finalize, shard_init,
                  shard_rank, shard_rms, unpack, unpack_aux, validate_dims)

__all__ = [
    "AUX_NAMES", "SAFARA_AUX_BT", "SAFARA_AUX_SP", "empty_aux", "rhs_aux", "rhs_norm",
    "rhs_slab_aux", "rhs_sumsq", "unpack_aux", "seismic_dz",
    "SAFARA_FLAG_STRICT", "SAFARA_PART_ALL", "SAFARA_PART_EDGE", "SAFARA_PART_INTERIOR",
    "Coeffs", "Dims", "SafaraError", "canonical_dims", "coeffs_nas", "empty_field", "init",
    "kernel_info", "launch_count", "pack", "pitch", "rhs", "rhs_host", "rhs_host_ex", "rhs_slab", "unpack",
    "validate_dims", "Peer", "rhs_peer", "ipc_get", "ipc_open", "ipc_close",
    "get_unique_id", "shard_init", "shard_finalize", "shard_rank", "rhs_sharded", "shard_rms",
    "rhs_rms", "strerror", "BtState", "bt_coeffs_nas", "rhs_fused",
]

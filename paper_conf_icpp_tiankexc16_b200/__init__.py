"""B200-native (sm_100a) NAS BT/SP ``compute_rhs`` -- thin Python binding.

The computation lives in ``libsafara_rhs.so`` (C ABI: include/safara.h);
this package only marshals torch tensors into that ABI.  PyTorch supplies
device memory, streams and process groups.  See DESIGN.md.
"""
from ._abi import (SAFARA_FLAG_STRICT, SAFARA_PART_ALL, SAFARA_PART_EDGE,
                   SAFARA_PART_INTERIOR, Coeffs, Dims, SafaraError)
from .rhs import (canonical_dims, coeffs_nas, empty_field, init, kernel_info,
                  launch_count, pack, pitch, rhs, rhs_host, rhs_slab, unpack,
                  validate_dims)

__all__ = [
    "SAFARA_FLAG_STRICT", "SAFARA_PART_ALL", "SAFARA_PART_EDGE", "SAFARA_PART_INTERIOR",
    "Coeffs", "Dims", "SafaraError", "canonical_dims", "coeffs_nas", "empty_field", "init",
    "kernel_info", "launch_count", "pack", "pitch", "rhs", "rhs_host", "rhs_slab", "unpack",
    "validate_dims",
]

"""Build the sm_100a shared library ``libsafara_rhs.so`` in-tree with nvcc.

Three translation units: the kernel compiled twice (``--fmad=true`` for the
production variant, ``--fmad=false`` for the STRICT variant) and the host ABI.
cudart is linked statically so the library has no runtime-version coupling
with the PyTorch wheel; the driver API (cuTensorMapEncodeTiled) is resolved at
run time through cudaGetDriverEntryPoint, so loading needs no libcuda.
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
BUILD = os.path.join(ROOT, "build")
LIB = os.path.join(PKG, "libsafara_rhs.so")

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC",
                 "-I" + INCLUDE, "-I" + CSRC]


def _nccl_include() -> str:
    """Directory of nccl.h for the NCCL types/prototypes of shard.cu (the
    library itself is dlopen()ed at run time: torch's copy in a torch process)."""
    try:
        import nvidia.nccl as _n  # the wheel torch loads libnccl.so.2 from
        for base in list(getattr(_n, "__path__", [])):
            inc = os.path.join(base, "include")
            if os.path.exists(os.path.join(inc, "nccl.h")):
                return inc
    except ImportError:
        pass
    return "/usr/include"


UNITS = [
    ("rhs_fast.cu", ["--fmad=true", "-Xptxas", "-v"]),
    ("rhs_strict.cu", ["--fmad=false", "-Xptxas", "-v"]),
    ("norm.cu", []),
    ("seismic.cu", ["-Xptxas", "-v"]),
    ("api.cu", []),
    ("shard.cu", ["-I" + _nccl_include()]),
    ("bt_solve.cu", ["--fmad=false", "-Xptxas", "-v"]),
]
DEPS = ["rhs_kernel.cuh", "rhs_ws.cuh", "rhs_variant.inc", "safara_internal.h"]


def _mtime(p):
    return os.path.getmtime(p) if os.path.exists(p) else 0.0


def build(force: bool = False, verbose: bool = False, extra: list[str] | None = None,
          out: str | None = None, objdir: str | None = None) -> str:
    """Compile (if stale) and return the path of libsafara_rhs.so (or ``out``;
    ``objdir`` keeps a variant build's objects apart from the default ones)."""
    objdir = objdir or BUILD
    os.makedirs(objdir, exist_ok=True)
    lib = out or LIB
    extra = list(extra or [])
    srcs = [os.path.join(CSRC, u) for u, _ in UNITS] + [os.path.join(CSRC, d) for d in DEPS]
    srcs.append(os.path.join(INCLUDE, "safara.h"))
    newest = max(_mtime(s) for s in srcs)
    if not force and _mtime(lib) >= newest and not extra:
        return lib
    objs = []
    ptxas_log = []
    for unit, flags in UNITS:
        obj = os.path.join(objdir, unit.replace(".cu", ".o"))
        cmd = [NVCC, *COMMON, *flags, *extra, "-c", os.path.join(CSRC, unit), "-o", obj]
        res = subprocess.run(cmd, capture_output=True, text=True)
        if res.returncode != 0:
            sys.stderr.write(res.stdout + res.stderr)
            raise RuntimeError(f"nvcc failed for {unit}")
        ptxas_log.append(f"== {unit} {' '.join(flags)}\n{res.stdout}{res.stderr}")
        objs.append(obj)
    tmp = lib + f".tmp{os.getpid()}"
    cmd = [NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs, "-ldl"]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        sys.stderr.write(res.stdout + res.stderr)
        raise RuntimeError("nvcc link failed")
    os.replace(tmp, lib)
    with open(os.path.join(BUILD, "ptxas.txt") if out is None else out + ".ptxas.txt", "w") as fh:
        fh.write("\n".join(ptxas_log))
    if verbose:
        print("\n".join(ptxas_log))
    return lib


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))

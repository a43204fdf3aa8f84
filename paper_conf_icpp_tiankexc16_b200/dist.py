"""z-slab domain decomposition for multi-GPU compute_rhs.

Rank r owns global planes [k0, k0+nzl), nzl = nz//p + (r < nz % p).  Its u
slab holds nzl+4 planes in the canonical layout: local plane 2+t is global
plane k0+t, planes 0-1 / nzl+2..nzl+3 are ghosts filled by the halo exchange
(2 planes from each neighbour: the dissipation stencil reaches k+-2).  forcing
and rhs slabs are rank-local (nzl planes).  The only communication on the path
is this point-to-point exchange; there is no collective.

The exchange is library code (include/safara.h safara_rhs_sharded): the
library owns an NCCL communicator (`NcclShard`: torch supplies only the process
group that broadcasts the NCCL unique id) and, per pass, runs the grouped
ncclSend/ncclRecv on its comm stream while PART_INTERIOR runs on the caller's
stream, joins, then runs PART_EDGE.  `halo_ops` / `halo_exchange` are the same
exchange pattern written with torch.distributed P2P; they exist for the CPU
(gloo) tests of the partition / neighbour logic.

SURVEY §8(f) f2, `rhs_fused`: no exchange at all.  The only values a slab
needs from a neighbour are the own (i, j) columns of the two planes beyond its
end (the zeta register window), so the kernel (safara_rhs_peer) loads them
straight from the neighbours' u slabs over NVLink.  `PeerHalo` maps the
neighbours' slabs and flag words into this process (CUDA IPC handles passed
through the process group) and numbers the passes (epochs) that the kernel's
release/acquire flags synchronise.
"""
from __future__ import annotations

from dataclasses import dataclass

import torch
import torch.distributed as dist

from ._abi import SAFARA_PEER_EPOCH_AUTO, SAFARA_PEER_WORDS, Peer

GHOST = 2


def partition(nz: int, p: int) -> list[tuple[int, int]]:
    """[(k0, nzl)] for ranks 0..p-1; every rank owns >= 2 planes."""
    if p < 1 or nz // p < GHOST:
        raise ValueError(f"cannot split nz={nz} into {p} slabs of >= {GHOST} planes")
    base, rem = divmod(nz, p)
    out, k0 = [], 0
    for r in range(p):
        n = base + (1 if r < rem else 0)
        out.append((k0, n))
        k0 += n
    return out


@dataclass
class Slab:
    rank: int
    world: int
    k0: int
    nzl: int
    nx: int
    ny: int
    nz: int
    u: torch.Tensor        # (nzl+4, 5, ny, sy)
    forcing: torch.Tensor  # (nzl, 5, ny, sy)
    rhs: torch.Tensor      # (nzl, 5, ny, sy)

    def owned_u(self) -> torch.Tensor:
        return self.u[GHOST:GHOST + self.nzl]


def make_slab(u_global: torch.Tensor, f_global: torch.Tensor, nx: int, rank: int, world: int,
              device=None) -> Slab:
    """Cut this rank's slab out of canonical global fields (ghosts zeroed)."""
    nz = u_global.shape[0]
    k0, nzl = partition(nz, world)[rank]
    dev = device if device is not None else u_global.device
    shape = tuple(u_global.shape[1:])
    u = torch.zeros((nzl + 2 * GHOST,) + shape, dtype=torch.float64, device=dev)
    u[GHOST:GHOST + nzl] = u_global[k0:k0 + nzl].to(dev)
    f = f_global[k0:k0 + nzl].to(dev).contiguous()
    r = torch.empty_like(f)
    return Slab(rank, world, k0, nzl, nx, u_global.shape[2], nz, u, f, r)


def halo_ops(s: Slab, group=None) -> list:
    """P2P ops exchanging 2 planes with each neighbour (no ghosts beyond the
    global grid: the first/last rank skip that side)."""
    ops = []
    u = s.u
    if s.rank > 0:
        prev = s.rank - 1
        ops.append(dist.P2POp(dist.isend, u[GHOST:2 * GHOST], prev, group))
        ops.append(dist.P2POp(dist.irecv, u[0:GHOST], prev, group))
    if s.rank < s.world - 1:
        nxt = s.rank + 1
        ops.append(dist.P2POp(dist.isend, u[s.nzl:s.nzl + GHOST], nxt, group))
        ops.append(dist.P2POp(dist.irecv, u[s.nzl + GHOST:s.nzl + 2 * GHOST], nxt, group))
    return ops


def halo_exchange(s: Slab, group=None) -> list:
    """Post the exchange; returns the work handles (wait() them)."""
    ops = halo_ops(s, group)
    return dist.batch_isend_irecv(ops) if ops else []


def broadcast_unique_id(rank: int, group=None, src: int = 0) -> bytes:
    """Rank ``src`` draws a fresh NCCL unique id through the library
    (safara_get_unique_id); every rank gets the same bytes through the torch
    process group (any backend: gloo on CPU, NCCL on GPUs)."""
    from .rhs import get_unique_id
    obj = [get_unique_id() if rank == src else None]
    dist.broadcast_object_list(obj, src=src, group=group)
    return obj[0]


class NcclShard:
    """This rank's library-owned NCCL communicator (safara_shard_init).

    torch.distributed is used once, to broadcast the unique id; every pass
    then runs through the C ABI (safara_rhs_sharded / safara_shard_rms)."""

    def __init__(self, rank: int, world: int, device: int, group=None):
        from .rhs import init, shard_init
        init(device)
        uid = broadcast_unique_id(rank, group)
        self.rank, self.world, self.device = rank, world, device
        self.handle = shard_init(uid, rank, world, device)

    def rhs(self, s: Slab, coeffs, strict: bool = False, stream=None) -> torch.Tensor:
        from .rhs import rhs_sharded as _rhs_sharded
        return _rhs_sharded(self.handle, s.u, s.forcing, s.rhs, s.nx, s.nz, s.k0, coeffs,
                            strict=strict, stream=stream)

    def rms(self, s: Slab, stream=None) -> torch.Tensor:
        from .rhs import shard_rms
        return shard_rms(self.handle, s.rhs, s.nx, s.nz, s.k0, stream=stream)

    def close(self):
        if self.handle:
            from .rhs import shard_finalize
            shard_finalize(self.handle)
            self.handle = 0


def rhs_sharded(s: Slab, coeffs, shard: NcclShard, strict: bool = False,
                stream=None) -> torch.Tensor:
    """One distributed pass through the library (safara_rhs_sharded): NCCL
    halo exchange on the shard's comm stream overlapped with the interior
    planes, then the edge planes."""
    return shard.rhs(s, coeffs, strict=strict, stream=stream)


# ---- the halo fused into the pass --------------------------

def neighbours(nz: int, p: int, rank: int) -> dict:
    """Which neighbours rank ``rank`` reads and where their slabs start.

    k0_lo / k0_hi: first global plane the lower / upper neighbour owns (None
    at the grid ends).  Plane k of a neighbour sits at its local u plane
    k - k0_nb + GHOST (the make_slab layout)."""
    parts = partition(nz, p)
    k0, nzl = parts[rank]
    return {"k0": k0, "nzl": nzl,
            "lo": rank - 1 if rank > 0 else None,
            "hi": rank + 1 if rank < p - 1 else None,
            "k0_lo": parts[rank - 1][0] if rank > 0 else None,
            "k0_hi": k0 + nzl if rank < p - 1 else None}


def peer_struct(nb: dict, u_lo: int | None, u_hi: int | None, flags: int | None,
                flags_lo: int | None, flags_hi: int | None, epoch: int) -> Peer:
    """safara_peer_t from raw device pointers (0/None = absent)."""
    pr = Peer()
    pr.u_lo = u_lo or None
    pr.u_hi = u_hi or None
    pr.k0_lo = nb["k0_lo"] if nb["k0_lo"] is not None else 0
    pr.k0_hi = nb["k0_hi"] if nb["k0_hi"] is not None else 0
    pr.flags = flags or None
    pr.flags_lo = (flags_lo or None) if epoch else None
    pr.flags_hi = (flags_hi or None) if epoch else None
    pr.epoch = int(epoch)
    return pr


def new_flags(device) -> torch.Tensor:
    """A rank's zeroed SAFARA_PEER_WORDS flag words."""
    return torch.zeros(SAFARA_PEER_WORDS, dtype=torch.int64, device=device)


class PeerHaloUnavailable(RuntimeError):
    """The fused peer halo cannot map a neighbour's slab (e.g. expandable
    segments): use the library's NCCL path (NcclShard / rhs_sharded)."""


def ipc_unavailable_reason() -> str:
    """Why cudaIpcGetMemHandle may refuse torch's allocations."""
    import os
    conf = os.environ.get("PYTORCH_CUDA_ALLOC_CONF", "") + os.environ.get(
        "PYTORCH_ALLOC_CONF", "")
    if "expandable_segments:True" in conf.replace(" ", ""):
        return ("PYTORCH_CUDA_ALLOC_CONF has expandable_segments:True: the caching allocator "
                "maps VMM segments, which CUDA IPC cannot export; unset it or use the NCCL halo")
    return ("the tensor is not in an IPC-exportable cudaMalloc allocation (VMM / expandable "
            "segment or a foreign allocator); use the NCCL halo")


class PeerHalo:
    """Peer mapping of the neighbours' u slabs and flag words (one per rank).

    Exports this rank's u slab and flags as CUDA IPC handles, gathers every
    rank's through the process group (all_gather_object) and maps the two
    neighbours'.  ``peer()`` returns the safara_peer_t of the next pass
    (epoch + 1; ``sync=False`` -> epoch 0, inputs static)."""

    def __init__(self, s: Slab, group=None):
        from ._abi import SafaraError
        from .rhs import ipc_get, ipc_open
        self.slab = s
        self.flags = new_flags(s.u.device)
        self.nb = neighbours(s.nz, s.world, s.rank)
        self._opened = []
        # Every rank reports success or its reason, so a rank that cannot
        # export never leaves the others blocked in the gather: all raise.
        try:
            mine = (ipc_get(s.u), ipc_get(self.flags))
        except SafaraError as e:
            mine = f"rank {s.rank}: {e} -- {ipc_unavailable_reason()}"
        allx = [None] * s.world
        dist.all_gather_object(allx, mine, group=group)
        bad = [x for x in allx if isinstance(x, str)]
        if bad:
            raise PeerHaloUnavailable("; ".join(bad))

        def open_(r):
            (hu, ou), (hf, of) = allx[r]
            pu, pf = ipc_open(hu, ou), ipc_open(hf, of)
            self._opened += [(pu, ou), (pf, of)]
            return pu, pf

        self.u_lo = self.f_lo = self.u_hi = self.f_hi = None
        if self.nb["lo"] is not None:
            self.u_lo, self.f_lo = open_(self.nb["lo"])
        if self.nb["hi"] is not None:
            self.u_hi, self.f_hi = open_(self.nb["hi"])
        self.epoch = 0

    def peer(self, sync: bool = True, auto: bool = False) -> Peer:
        """safara_peer_t of the next pass.  auto: the epoch is counted on the
        device (SAFARA_PEER_EPOCH_AUTO), for passes captured in a CUDA graph."""
        if auto:
            return peer_struct(self.nb, self.u_lo, self.u_hi, self.flags.data_ptr(), self.f_lo,
                               self.f_hi, SAFARA_PEER_EPOCH_AUTO)
        if sync:
            self.epoch += 1
        return peer_struct(self.nb, self.u_lo, self.u_hi, self.flags.data_ptr(), self.f_lo,
                           self.f_hi, self.epoch if sync else 0)

    def timeouts(self) -> int:
        from ._abi import SAFARA_PEER_TIMEOUTS
        return int(self.flags[SAFARA_PEER_TIMEOUTS].item())

    def close(self):
        from .rhs import ipc_close
        for ptr, off in self._opened:
            ipc_close(ptr, off)
        self._opened = []


def rhs_fused(s: Slab, halo: PeerHalo, coeffs, strict: bool = False, sync: bool = True,
              stream=None, auto: bool = False) -> torch.Tensor:
    """One distributed pass, halo fused into the kernel (one launch, no
    exchange): f2.  Do not mix host-numbered (sync) and device-numbered
    (auto) epochs on one PeerHalo."""
    from .rhs import rhs_peer
    rhs_peer(s.u, s.forcing, s.rhs, s.nx, s.nz, s.k0, halo.peer(sync, auto), coeffs,
             strict=strict, stream=stream)
    return s.rhs

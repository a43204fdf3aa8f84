"""z-slab domain decomposition for multi-GPU compute_rhs.

Rank r owns global planes [k0, k0+nzl), nzl = nz//p + (r < nz % p).  Its u
slab holds nzl+4 planes in the canonical layout: local plane 2+t is global
plane k0+t, planes 0-1 / nzl+2..nzl+3 are ghosts filled by the halo exchange
(2 planes from each neighbour: the dissipation stencil reaches k+-2).  forcing
and rhs slabs are rank-local (nzl planes).  The only communication on the path
is this point-to-point exchange; there is no collective.

The exchange uses torch.distributed P2P (NCCL over NVLink on GPUs, gloo on CPU
for tests).  `rhs_sharded` overlaps it with the ghost-independent planes:
PART_INTERIOR runs on the compute stream while the exchange is in flight,
PART_EDGE after the exchange completes.
"""
from __future__ import annotations

from dataclasses import dataclass

import torch
import torch.distributed as dist

from ._abi import SAFARA_PART_EDGE, SAFARA_PART_INTERIOR

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


def rhs_sharded(s: Slab, coeffs, comm_stream: torch.cuda.Stream | None = None,
                strict: bool = False, group=None) -> torch.Tensor:
    """One distributed pass: exchange overlapped with the interior planes."""
    from .rhs import rhs_slab
    compute = torch.cuda.current_stream()
    comm = comm_stream or torch.cuda.Stream()
    comm.wait_stream(compute)  # u is ready
    with torch.cuda.stream(comm):
        works = halo_exchange(s, group)
    rhs_slab(s.u, s.forcing, s.rhs, s.nx, s.nz, s.k0, coeffs, part=SAFARA_PART_INTERIOR,
             strict=strict, stream=compute)
    for w in works:
        w.wait()                # compute stream waits for the ghosts
    compute.wait_stream(comm)
    rhs_slab(s.u, s.forcing, s.rhs, s.nx, s.nz, s.k0, coeffs, part=SAFARA_PART_EDGE,
             strict=strict, stream=compute)
    return s.rhs

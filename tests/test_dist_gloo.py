"""Host logic of the z-slab decomposition on CPU: partitioning and the 2-plane
halo exchange over torch.distributed (gloo, world sizes 2 and 3)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icpp_tiankexc16_b200 import dist as sd


def test_partition():
    assert sd.partition(162, 8) == [(0, 21), (21, 21), (42, 20), (62, 20), (82, 20), (102, 20),
                                    (122, 20), (142, 20)]
    assert sd.partition(102, 8)[-1] == (90, 12)
    for nz, p in ((12, 2), (36, 3), (41, 4), (162, 8), (16, 8)):
        parts = sd.partition(nz, p)
        assert sum(n for _, n in parts) == nz
        assert all(n >= 2 for _, n in parts)
        assert all(parts[i][0] + parts[i][1] == parts[i + 1][0] for i in range(p - 1))
    with pytest.raises(ValueError):
        sd.partition(5, 3)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, nz, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import nasgen
        import paper_conf_icpp_tiankexc16_b200 as sr
        inp = nasgen.make_inputs(13, 10, nz, seed=7, dt=0.001)
        ug = sr.pack(inp.u, device="cpu")
        fg = sr.pack(inp.forcing, device="cpu")
        s = sd.make_slab(ug, fg, 13, rank, world, device="cpu")
        for w in sd.halo_exchange(s):
            w.wait()
        ok = True
        g = sd.GHOST
        if rank > 0:
            ok &= torch.equal(s.u[0:g], ug[s.k0 - g:s.k0])
        else:
            ok &= bool((s.u[0:g] == 0).all())
        if rank < world - 1:
            ok &= torch.equal(s.u[g + s.nzl:], ug[s.k0 + s.nzl:s.k0 + s.nzl + g])
        ok &= torch.equal(s.owned_u(), ug[s.k0:s.k0 + s.nzl])
        ok &= torch.equal(s.forcing, fg[s.k0:s.k0 + s.nzl])
        q.put((rank, bool(ok)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,nz", [(2, 12), (3, 17), (2, 7)])
def test_halo_exchange_gloo(world, nz):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, nz, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    res = dict(q.get(timeout=10) for _ in range(world))
    assert all(p.exitcode == 0 for p in procs)
    assert all(res[r] for r in range(world)), res

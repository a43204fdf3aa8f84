"""the halo fused into the pass (safara_rhs_peer).

Each z-slab's kernel reads the own columns of the two planes beyond its ends
straight from the neighbours' u slabs (peer pointers), with no exchange step.
Bar: STRICT bit-identical to the CPU oracle (and production bit-identical to
the single-GPU production pass: the same kernel body computes every plane),
at every partition, with the ghost planes of every u slab poisoned (NaN) to
prove they are never read.

The GPU box has one GPU, so "ranks" are slabs on the same device:
  * in-process: peer pointers are the other slabs' device addresses; with
    epoch > 0 the kernels run concurrently on separate streams (small grids:
    all CTAs co-resident) and synchronise through the flag words;
  * two processes: the slabs are mapped through CUDA IPC handles exchanged
    over a gloo process group (the PeerHalo path the multi-GPU bench uses).
"""
import os

import numpy as np
import pytest
import torch

import nasgen
import oracle
import paper_conf_icpp_tiankexc16_b200 as sr
from paper_conf_icpp_tiankexc16_b200 import dist as sd
from paper_conf_icpp_tiankexc16_b200._abi import (SAFARA_PEER_ARRIVED, SAFARA_PEER_HI_DONE,
                                                  SAFARA_PEER_HI_READY, SAFARA_PEER_LO_DONE,
                                                  SAFARA_PEER_LO_READY, SAFARA_PEER_TIMEOUTS)

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _init():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    sr.init(0)


def _slabs(inp, p):
    nz, ny, nx, _ = inp.u.shape
    ug, fg = sr.pack(inp.u, device="cpu"), sr.pack(inp.forcing, device="cpu")
    slabs = []
    for r in range(p):
        s = sd.make_slab(ug, fg, nx, r, p, device="cuda")
        s.u[:sd.GHOST] = float("nan")       # ghosts are never read by the fused path
        s.u[-sd.GHOST:] = float("nan")
        s.rhs.fill_(float("nan"))
        slabs.append(s)
    return slabs


def _peers(slabs, flags, epoch):
    out = []
    for r, s in enumerate(slabs):
        nb = sd.neighbours(s.nz, len(slabs), r)
        lo, hi = nb["lo"], nb["hi"]
        out.append(sd.peer_struct(
            nb, slabs[lo].u.data_ptr() if lo is not None else None,
            slabs[hi].u.data_ptr() if hi is not None else None,
            flags[r].data_ptr() if flags else None,
            flags[lo].data_ptr() if flags and lo is not None else None,
            flags[hi].data_ptr() if flags and hi is not None else None, epoch))
    return out


def _gather(slabs, nx):
    return np.concatenate([sr.unpack(s.rhs, nx) for s in slabs], axis=0)


def assert_tol(g, o, rtol=1e-12, atol=1e-14):
    err = np.abs(g - o)
    bound = rtol * np.abs(o) + atol
    assert not (err > bound).any() and not np.isnan(g).any(), \
        f"worst ratio {np.nanmax(err / bound):.3g}"


def _c(inp):
    nz, ny, nx, _ = inp.u.shape
    return sr.coeffs_nas(nx, ny, nz, inp.dt)


@pytest.mark.parametrize("shape,p", [((9, 13, 37), 2), ((23, 15, 40), 3), ((12, 12, 12), 3),
                                     ((24, 34, 30), 4), ((36, 36, 36), 8), ((17, 29, 37), 5)])
@pytest.mark.parametrize("strict", [True, False])
def test_peer_slabs_sequential(shape, p, strict):
    """epoch 0 (static inputs): slabs one after another on one stream."""
    nz, ny, nx = shape
    inp = nasgen.make_inputs(nx, ny, nz, seed=4, B=1e-2, dt=0.002)
    slabs = _slabs(inp, p)
    c = _c(inp)
    for s, pr in zip(slabs, _peers(slabs, None, 0)):
        sr.rhs_peer(s.u, s.forcing, s.rhs, nx, nz, s.k0, pr, c, strict=strict)
    torch.cuda.synchronize()
    g = _gather(slabs, nx)
    o = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=8)
    if strict:
        assert np.array_equal(g, o), f"max |g-o| = {np.nanmax(np.abs(g - o)):.3g}"
    else:
        assert_tol(g, o)


@pytest.mark.parametrize("p", [2, 8])
def test_peer_full_class_c(p):
    """BT class C in the multi-GPU bench's launch configuration (production):
    every slab within the tolerance of the oracle (a plane's position in the
    3-step unrolled march depends on the partition, and each unrolled copy
    may be FMA-contracted differently, so production is not bitwise across
    partitions -- SURVEY §8(c) pin P8)."""
    inp = nasgen.make_class("BT", "C", seed=1)
    n = inp.u.shape[0]
    slabs = _slabs(inp, p)
    for s, pr in zip(slabs, _peers(slabs, None, 0)):
        sr.rhs_peer(s.u, s.forcing, s.rhs, n, n, s.k0, pr, _c(inp))
    torch.cuda.synchronize()
    assert_tol(_gather(slabs, n), oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=16))


def _concurrent_pass(slabs, flags, epoch, c, nx, strict, streams, delay_rank=None,
                     restore=None):
    peers = _peers(slabs, flags, epoch)
    for r, (s, pr) in enumerate(zip(slabs, peers)):
        with torch.cuda.stream(streams[r]):
            if r == delay_rank:
                # this rank's u becomes final only after a ~1 ms spin: its
                # neighbours must wait for its READY word, not read early
                torch.cuda._sleep(2_000_000)
                s.u.copy_(restore)
            sr.rhs_peer(s.u, s.forcing, s.rhs, nx, s.nz, s.k0, pr, c, strict=strict,
                        stream=streams[r])
            if r == delay_rank:
                # ...and its grid completes only after the neighbours read it
                s.u[sd.GHOST:-sd.GHOST] = float("nan")
    torch.cuda.synchronize()


# The concurrent tests run in a fresh process with CUDA_DEVICE_MAX_CONNECTIONS
# = 32 and eager module loading.  With the default 8 hardware queues two of
# the simulated ranks' streams can share one queue, and with lazy loading the
# first launch of a not-yet-loaded kernel (e.g. torch's sleep or fill kernel)
# waits for the kernels already running; either way a rank whose kernel waits
# for a neighbour could then hold that neighbour back until its wait gives up
# -- an artefact of simulating ranks on one GPU, not of the protocol (one GPU
# per rank in production, where a rank only ever waits for other GPUs).
_CHILD_ENV = {"CUDA_DEVICE_MAX_CONNECTIONS": "32", "CUDA_MODULE_LOADING": "EAGER"}


def _in_child(fn, *args):
    import torch.multiprocessing as mp
    old = {k: os.environ.get(k) for k in _CHILD_ENV}
    os.environ.update(_CHILD_ENV)
    try:
        ctx = mp.get_context("spawn")
        q = ctx.Queue()
        pr = ctx.Process(target=_child_main, args=(fn, args, q))
        pr.start()
        ok, msg = q.get(timeout=600)
        pr.join(timeout=60)
    finally:
        for k, v in old.items():
            if v is None:
                del os.environ[k]
            else:
                os.environ[k] = v
    assert ok, msg


def _child_main(fn, args, q):
    import traceback
    try:
        sr.init(0)
        fn(*args)
        q.put((True, ""))
    except BaseException:
        q.put((False, traceback.format_exc()))


def _epochs_body(shape, p):
    nz, ny, nx = shape
    inp = nasgen.make_inputs(nx, ny, nz, seed=5, B=1e-2, dt=0.002)
    o = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=8)
    slabs = _slabs(inp, p)
    flags = [sd.new_flags("cuda") for _ in range(p)]
    streams = [torch.cuda.Stream() for _ in range(p)]
    c = _c(inp)
    for epoch in (1, 2, 3):
        for s in slabs:
            s.rhs.fill_(float("nan"))
        torch.cuda.synchronize()
        _concurrent_pass(slabs, flags, epoch, c, nx, True, streams)
        assert np.array_equal(_gather(slabs, nx), o), f"epoch {epoch}"
        for r, f in enumerate(flags):
            f = f.cpu().tolist()
            assert f[SAFARA_PEER_TIMEOUTS] == 0 and f[SAFARA_PEER_ARRIVED] == 0, f
            if r > 0:
                assert f[SAFARA_PEER_LO_READY] == epoch and f[SAFARA_PEER_LO_DONE] == epoch
            if r < p - 1:
                assert f[SAFARA_PEER_HI_READY] == epoch and f[SAFARA_PEER_HI_DONE] == epoch


@pytest.mark.parametrize("shape,p", [((24, 34, 30), 2), ((24, 34, 30), 4), ((20, 14, 40), 3)])
def test_peer_epochs_concurrent(shape, p):
    """epoch > 0: all ranks' kernels in flight together, three passes, flag
    protocol checked (no timeouts, counters reset, READY/DONE = epoch)."""
    _in_child(_epochs_body, shape, p)


def _auto_graph_body(shape, p):
    """SAFARA_PEER_EPOCH_AUTO: each rank captures 3 passes into its own CUDA
    graph (the same peer struct in every node); the graphs replay
    concurrently, twice, and the device epoch counter advances to 6."""
    from paper_conf_icpp_tiankexc16_b200._abi import SAFARA_PEER_EPOCH_AUTO, SAFARA_PEER_EPOCH_WORD
    nz, ny, nx = shape
    inp = nasgen.make_inputs(nx, ny, nz, seed=8, B=1e-2, dt=0.002)
    o = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=8)
    slabs = _slabs(inp, p)
    flags = [sd.new_flags("cuda") for _ in range(p)]
    streams = [torch.cuda.Stream() for _ in range(p)]
    peers = _peers(slabs, flags, SAFARA_PEER_EPOCH_AUTO)
    c = _c(inp)
    torch.cuda._sleep(1000)
    torch.cuda.synchronize()
    graphs = []
    for r, (s, pr) in enumerate(zip(slabs, peers)):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=streams[r]):
            for _ in range(3):
                sr.rhs_peer(s.u, s.forcing, s.rhs, nx, nz, s.k0, pr, c, strict=True,
                            stream=streams[r])
        graphs.append(g)
    torch.cuda.synchronize()
    for rep in range(2):
        for s in slabs:
            s.rhs.fill_(float("nan"))
        torch.cuda.synchronize()
        for r, g in enumerate(graphs):
            with torch.cuda.stream(streams[r]):
                g.replay()
        torch.cuda.synchronize()
        assert np.array_equal(_gather(slabs, nx), o), f"replay {rep}"
    for f in flags:
        f = f.cpu().tolist()
        assert f[SAFARA_PEER_TIMEOUTS] == 0 and f[SAFARA_PEER_ARRIVED] == 0, f
        assert f[SAFARA_PEER_EPOCH_WORD] == 6, f


@pytest.mark.parametrize("shape,p", [((24, 34, 30), 2), ((20, 14, 40), 3)])
def test_peer_auto_epoch_graphs(shape, p):
    _in_child(_auto_graph_body, shape, p)


def _waits_body():
    nz, ny, nx = 30, 34, 24
    p, mid = 3, 1
    inp = nasgen.make_inputs(nx, ny, nz, seed=6, B=1e-2, dt=0.002)
    o = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=8)
    slabs = _slabs(inp, p)
    good = slabs[mid].u.clone()
    slabs[mid].u[sd.GHOST:-sd.GHOST] = float("nan")
    flags = [sd.new_flags("cuda") for _ in range(p)]
    streams = [torch.cuda.Stream() for _ in range(p)]
    torch.cuda._sleep(1000)  # every kernel of the pass is loaded before it starts
    torch.cuda.synchronize()
    _concurrent_pass(slabs, flags, 1, _c(inp), nx, True, streams, delay_rank=mid, restore=good)
    fl = [f.cpu().tolist() for f in flags]
    assert all(f[SAFARA_PEER_TIMEOUTS] == 0 for f in fl), fl
    assert np.array_equal(_gather(slabs, nx), o)


def test_peer_waits_for_neighbour():
    """The middle rank's u is NaN until a delayed copy on its own stream and
    is NaN-poisoned right after its pass: its neighbours must read it in
    between (READY acquire before, DONE before its grid completes)."""
    _in_child(_waits_body)


def test_peer_argument_errors():
    inp = nasgen.make_inputs(12, 12, 12, seed=1)
    slabs = _slabs(inp, 2)
    c = _c(inp)
    s0, s1 = slabs
    ok = _peers(slabs, None, 0)
    # rank 0 must not have a lower neighbour
    bad = sd.peer_struct(sd.neighbours(12, 2, 0), s1.u.data_ptr(), s1.u.data_ptr(), None, None,
                         None, 0)
    with pytest.raises(sr.SafaraError):
        sr.rhs_peer(s0.u, s0.forcing, s0.rhs, 12, 12, s0.k0, bad, c)
    # rank 1 needs its lower neighbour
    bad = sd.peer_struct(sd.neighbours(12, 2, 1), None, None, None, None, None, 0)
    with pytest.raises(sr.SafaraError):
        sr.rhs_peer(s1.u, s1.forcing, s1.rhs, 12, 12, s1.k0, bad, c)
    # epoch > 0 needs flag words
    bad = sd.peer_struct(sd.neighbours(12, 2, 1), s0.u.data_ptr(), None, None, None, None, 3)
    with pytest.raises(sr.SafaraError):
        sr.rhs_peer(s1.u, s1.forcing, s1.rhs, 12, 12, s1.k0, bad, c)
    # inconsistent neighbour start
    pr = ok[1]
    pr.k0_lo = s1.k0 - 1
    with pytest.raises(sr.SafaraError):
        sr.rhs_peer(s1.u, s1.forcing, s1.rhs, 12, 12, s1.k0, pr, c)


# ---- two processes, CUDA IPC (the PeerHalo path) ------------------------------

def _ipc_worker(rank, world, port, shape, sync, out_q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        sr.init(0)
        nz, ny, nx = shape
        inp = nasgen.make_inputs(nx, ny, nz, seed=7, B=1e-2, dt=0.002)
        ug, fg = sr.pack(inp.u, device="cpu"), sr.pack(inp.forcing, device="cpu")
        s = sd.make_slab(ug, fg, nx, rank, world, device="cuda")
        s.u[:sd.GHOST] = float("nan")
        s.u[-sd.GHOST:] = float("nan")
        halo = sd.PeerHalo(s)
        c = sr.coeffs_nas(nx, ny, nz, inp.dt)
        torch.cuda.synchronize()
        dist.barrier()
        for _ in range(3):
            sd.rhs_fused(s, halo, c, strict=True, sync=sync)
        torch.cuda.synchronize()
        dist.barrier()          # nobody unmaps while a neighbour still reads
        res = (rank, sr.unpack(s.rhs, nx), halo.timeouts())
        halo.close()
        out_q.put(res)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("sync", [False, True])
def test_peer_two_processes_ipc(sync):
    import socket

    import torch.multiprocessing as mp
    shape = (20, 14, 24)
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, shape, sync, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = sorted([q.get(timeout=300) for _ in procs], key=lambda t: t[0])
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    nz, ny, nx = shape
    inp = nasgen.make_inputs(nx, ny, nz, seed=7, B=1e-2, dt=0.002)
    o = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=8)
    assert all(t[2] == 0 for t in res), "peer waits timed out"
    assert np.array_equal(np.concatenate([t[1] for t in res], axis=0), o)

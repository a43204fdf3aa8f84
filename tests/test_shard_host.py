"""Host side of the sharded C ABI (include/safara.h
safara_get_unique_id / safara_shard_init / safara_rhs_sharded /
safara_shard_rms / safara_shard_finalize) without a GPU: argument checks
(the paper's up-front clause validation, returns error
codes instead of running anything), the NCCL unique id, and its round trip
through a torch process group (gloo, world size 2)."""
import ctypes
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import paper_conf_icpp_tiankexc16_b200 as sr
from paper_conf_icpp_tiankexc16_b200 import _abi, build
from paper_conf_icpp_tiankexc16_b200 import dist as sd

ERR_ARG, ERR_SHAPE, ERR_NO_DEVICE, ERR_NCCL = -1, -2, -8, -9


@pytest.fixture(scope="module")
def L():
    build.build()
    return _abi.lib()


def test_unique_id_bytes(L):
    a, b = sr.get_unique_id(), sr.get_unique_id()
    assert isinstance(a, bytes) and len(a) == _abi.SAFARA_UNIQUE_ID_BYTES == 128
    assert a != b                      # fresh bootstrap handle per call
    assert L.safara_get_unique_id(None) == ERR_ARG


def test_shard_init_argument_checks(L):
    uid = sr.get_unique_id()
    h = ctypes.c_void_p()
    assert L.safara_shard_init(None, 0, 1, 0, ctypes.byref(h)) == ERR_ARG
    assert L.safara_shard_init(uid, 0, 1, 0, None) == ERR_ARG
    assert L.safara_shard_init(uid, 1, 1, 0, ctypes.byref(h)) == ERR_ARG   # rank >= nranks
    assert L.safara_shard_init(uid, -1, 2, 0, ctypes.byref(h)) == ERR_ARG
    assert L.safara_shard_init(uid, 0, 0, 0, ctypes.byref(h)) == ERR_ARG
    if not torch.cuda.is_available():
        # valid arguments, no device: the sm_100 check fails, nothing is created
        assert L.safara_shard_init(uid, 0, 1, 0, ctypes.byref(h)) == ERR_NO_DEVICE
        assert not h.value


def test_sharded_calls_reject_bad_handles(L):
    d = sr.canonical_dims(12, 12, 12)
    c = sr.coeffs_nas(12, 12, 12, 0.01)
    bogus = ctypes.create_string_buffer(64)     # not a handle from safara_shard_init
    for h in (None, ctypes.addressof(bogus)):
        assert L.safara_rhs_sharded(h, 16, 16, 16, 12, 12, 12, 0, 12, ctypes.byref(c),
                                    None) == ERR_ARG
        assert L.safara_rhs_sharded_ex(h, 16, 16, 16, ctypes.byref(d), 0, 12, ctypes.byref(c),
                                       0, None) == ERR_ARG
        assert L.safara_shard_rms(h, 16, ctypes.byref(d), 0, 12, 16, 16, None) == ERR_ARG
        r, n = ctypes.c_int(), ctypes.c_int()
        assert L.safara_shard_rank(h, ctypes.byref(r), ctypes.byref(n)) == ERR_ARG
        assert L.safara_shard_finalize(h) == ERR_ARG


def test_error_strings(L):
    assert "NCCL" in sr.strerror(ERR_NCCL)
    for code in (0, -1, -2, -3, -4, -5, -6, -7, -8, -9):
        assert sr.strerror(code) != "unknown error code"


def test_header_documents_the_sharded_calls():
    syms = _abi.header_symbols()
    for s in ("safara_get_unique_id", "safara_shard_init", "safara_rhs_sharded",
              "safara_rhs_sharded_ex", "safara_shard_rms", "safara_shard_rank",
              "safara_shard_finalize", "safara_rhs_rms"):
        assert s in syms, s


def test_python_shape_checks_on_host_tensors():
    """The wrappers check shapes before any pointer reaches the C side
    (the descriptor alone sizes the TMA maps and stores)."""
    from paper_conf_icpp_tiankexc16_b200.rhs import _canonical_fields
    p = sr.pitch(12)
    u = torch.zeros((12, 5, 12, p), dtype=torch.float64)
    assert _canonical_fields(12, ((u, "u"), (u, "f"), (u, "r"))) == (12, 12)
    with pytest.raises(ValueError):
        _canonical_fields(12, ((u, "u"), (torch.zeros((11, 5, 12, p)), "f"), (u, "r")))
    with pytest.raises(ValueError):   # pitch != pitch(nx)
        _canonical_fields(12, ((u, "u"), (torch.zeros((12, 5, 12, 12)), "f"), (u, "r")))
    slab_u = torch.zeros((6 + 4, 5, 12, p))
    slab_f = torch.zeros((6, 5, 12, p))
    assert _canonical_fields(12, ((slab_u, "u"), (slab_f, "f"), (slab_f, "r")),
                             nplanes_u=10) == (6, 12)
    with pytest.raises(ValueError):   # u slab without its 4 ghost planes
        _canonical_fields(12, ((slab_f, "u"), (slab_f, "f"), (slab_f, "r")), nplanes_u=10)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _uid_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        uid = sd.broadcast_unique_id(rank)
        q.put((rank, uid))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_unique_id_round_trip_gloo(world):
    """Rank 0's id reaches every rank byte for byte through the process group
    (the only thing torch.distributed does for the sharded path)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_uid_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert len(got[0]) == 128
    assert all(got[r] == got[0] for r in range(world))

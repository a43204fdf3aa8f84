"""Multi-GPU arm of bench.py (torchrun, one rank per GPU, NCCL): BT class C
split into z-slabs, one compute_rhs pass per step.  --halo peer (default):
the halo is fused into the kernel (safara_rhs_peer: one
launch per rank per pass, neighbours' planes loaded over NVLink, epoch flags);
--halo nccl: the library's NCCL send/recv exchange overlapped with the
interior planes (safara_rhs_sharded on a library-owned communicator, SURVEY
§8(b)/(e)).

Timing: barrier + synchronize on both sides of the K timed steps, CUDA events
on each rank's compute stream, MAX over ranks (all_reduce).  value = all grid
points / that time (strong scaling: the grid is fixed).
"""
from __future__ import annotations

import json
import os
import time

import torch
import torch.distributed as dist


def run(args):
    import nasgen

    from . import dist as sd
    from bench import ClockSampler, measured_peaks

    from .rhs import coeffs_nas, init, kernel_info, launch_count, pack

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", str(rank)))
    # SAFARA_SAME_GPU=1: every rank on GPU 0 with a gloo group -- a functional
    # check of the whole multi-process path (IPC mapping, epochs, e2e, JSON)
    # on a one-GPU box; its timings are time-sliced and mean nothing.
    same_gpu = os.environ.get("SAFARA_SAME_GPU") == "1"
    if world == 1:  # bench.py --dist without torchrun
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29511")
    if same_gpu:
        local = 0
        if args.halo == "nccl" and world > 1:
            # NCCL itself refuses two ranks of one communicator on one device
            raise SystemExit("SAFARA_SAME_GPU=1 supports only --halo peer: NCCL does not allow "
                             "two ranks on one GPU (the NCCL halo needs one GPU per rank)")
    torch.cuda.set_device(local)
    if same_gpu:
        dist.init_process_group("gloo", rank=rank, world_size=world)
    else:
        dist.init_process_group("nccl", rank=rank, world_size=world,
                                device_id=torch.device("cuda", local))
    cdev = "cpu" if same_gpu else "cuda"  # collectives' tensors
    init(local)
    bench, cls = args.config.split("-")
    n, dt = nasgen.CLASSES[(bench, cls)]
    inp = nasgen.make_class(bench, cls, seed=1)
    ug, fg = pack(inp.u, device="cpu"), pack(inp.forcing, device="cpu")
    s = sd.make_slab(ug, fg, n, rank, world, device=f"cuda:{local}")
    c = coeffs_nas(n, n, n, dt)
    compute = torch.cuda.current_stream()
    def all_ok(ok: bool) -> bool:
        """Every rank succeeded (collective agreement on a local outcome)."""
        f = torch.tensor([0 if ok else 1], device=cdev)
        dist.all_reduce(f, op=dist.ReduceOp.MAX)
        return int(f.item()) == 0

    halo, note = None, None
    if args.halo == "peer":
        # the fused halo needs CUDA IPC + peer access between the ranks' GPUs;
        # if any rank cannot map its neighbours, every rank uses the NCCL halo
        try:
            halo = sd.PeerHalo(s)
            ok = True
        except Exception as e:  # noqa: BLE001 -- reported in the JSON line
            ok, note = False, f"peer halo unavailable ({type(e).__name__}: {e}); NCCL halo used"
        if not all_ok(ok):
            if halo is not None:
                halo.close()
            halo = None
            note = note or "a peer rank could not map its neighbours; NCCL halo used"

    shard = None
    if halo is None:
        # the library owns the communicator; torch only broadcasts its id
        shard = sd.NcclShard(rank, world, local)

    use_graph = args.graph > 0 and halo is not None
    auto_epochs = use_graph  # fixed for the run: never mix host and device epoch numbering

    def step(st=None):
        if halo is not None:
            # graph mode: device-counted epochs (the same struct replays)
            sd.rhs_fused(s, halo, c, strict=args.strict, stream=st or compute, auto=auto_epochs)
        else:
            sd.rhs_sharded(s, c, shard, strict=args.strict, stream=st or compute)

    if use_graph:
        # G passes per CUDA graph (one launch gap per G passes); every rank
        # captures and replays the same count, epochs advance on the device
        for _ in range(3):
            step()
        torch.cuda.synchronize()
        graph = torch.cuda.CUDAGraph()
        g0 = launch_count()
        try:
            with torch.cuda.graph(graph):
                for _ in range(args.graph):
                    step(torch.cuda.current_stream())
            ok = True
        except Exception as e:  # noqa: BLE001 -- reported in the JSON line
            ok, note = False, f"graph capture failed ({type(e).__name__}); stream launches used"
        per_graph = launch_count() - g0
        torch.cuda.synchronize()
        eager_step = step
        if all_ok(ok):
            G = args.graph
            args.steps = max(G, (args.steps // G) * G)
            dist.barrier()

            def step(st=None):  # noqa: F811 -- one replay = G passes
                graph.replay()
        else:
            use_graph = False
            note = note or "graph capture failed on a peer rank; stream launches used"

    w0, w1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    w0.record(compute)
    nstep = (lambda k: max(1, k // args.graph)) if use_graph else (lambda k: k)
    for _ in range(nstep(max(args.warmup, 3))):
        step()
    w1.record(compute)
    torch.cuda.synchronize()
    # untimed soak so the clock sampler sees the loaded GPU; every rank runs
    # the same number of passes (the peer halo pairs epochs across ranks)
    wms = torch.tensor([w0.elapsed_time(w1) / nstep(max(args.warmup, 3))], device=cdev)
    dist.all_reduce(wms, op=dist.ReduceOp.MAX)
    nsoak = int(min(20000, args.soak_s * 1e3 / max(wms.item(), 1e-3)))
    dist.barrier()
    sampler = None
    if rank == 0:
        sampler = ClockSampler(local)
        sampler.start()
    for t in range(nsoak):
        step()
        if t % 50 == 49:
            torch.cuda.synchronize()
    torch.cuda.synchronize()
    dist.barrier()
    l0 = launch_count()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(compute)
    for _ in range(nstep(args.steps)):
        step()
    e1.record(compute)
    torch.cuda.synchronize()
    dist.barrier()
    ms = torch.tensor([e0.elapsed_time(e1)], device=cdev)
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    launches = torch.tensor([launch_count() - l0 + (per_graph * nstep(args.steps) if use_graph
                                                    else 0)], device=cdev, dtype=torch.int64)
    dist.all_reduce(launches)
    ms_per_step = ms.item() / args.steps
    pts = n ** 3
    value = pts / (ms_per_step * 1e-3) / 1e9

    # e2e through the public API: pinned host slab -> device, pass, rhs -> host
    hu = s.u.cpu().pin_memory()
    hf = s.forcing.cpu().pin_memory()
    hr = torch.empty(s.rhs.shape, dtype=torch.float64).pin_memory()
    torch.cuda.synchronize()
    dist.barrier()
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    t0.record(compute)
    for _ in range(args.e2e_steps):
        s.u.copy_(hu, non_blocking=True)
        s.forcing.copy_(hf, non_blocking=True)
        (eager_step if use_graph else step)()
        hr.copy_(s.rhs, non_blocking=True)
    t1.record(compute)
    torch.cuda.synchronize()
    dist.barrier()
    ems = torch.tensor([t0.elapsed_time(t1) / args.e2e_steps], device=cdev)
    dist.all_reduce(ems, op=dist.ReduceOp.MAX)
    io = torch.tensor([(hu.numel() + hf.numel()) * 8, hr.numel() * 8,
                       halo.timeouts() if halo is not None else 0], device=cdev,
                      dtype=torch.int64)
    dist.all_reduce(io)
    clocks = ClockSampler.summarise(sampler.stop()) if sampler is not None else None
    if halo is not None:
        torch.cuda.synchronize()
        dist.barrier()          # nobody unmaps a slab a neighbour may still read
        halo.close()
    if shard is not None:
        torch.cuda.synchronize()
        shard.close()

    if rank == 0:
        peak, peak_kind = measured_peaks()
        achieved = 120 * pts / (ms_per_step * 1e-3) / 1e9
        line = {
            "metric": "rhs grid-points/s", "value": value, "unit": "Gpt/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": nasgen.config_name(bench, cls), "grid": [n, n, n],
                       "points": pts,
                       "parallelism": (f"z-slab x{world}, halo fused into the kernel (NVLink "
                                       "peer loads, epoch flags)" + (
                                           f", CUDA graph of {args.graph} passes" if use_graph
                                           else "") if halo is not None else
                                       f"z-slab x{world}, 2-plane NCCL send/recv halo "
                                       "(library-owned communicator)"),
                       "variant": "strict" if args.strict else "production",
                       "l2": "per-rank slabs; inputs > L2 at C/1-2, no flush"},
            "hbm_gbs": achieved,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak * world,
                         "unit": "GB/s", "frac": achieved / (peak * world),
                         "peak_kind": f"{peak_kind} per-GPU x {world}", "traffic": None,
                         "bytes_per_point": 120, "kernel_ms": ms_per_step},
            "clocks": clocks,
            "e2e": {"value": pts / (ems.item() * 1e-3) / 1e9, "unit": "Gpt/s",
                    "h2d_bytes_per_step": int(io[0].item()),
                    "d2h_bytes_per_step": int(io[1].item()),
                    "note": "every rank copies its slab (u incl. ghosts, forcing) in and rhs out"},
            "gpu_launches": int(launches.item()),
            "peer_wait_timeouts": int(io[2].item()),
            "note": note,
            "kernel": kernel_info(args.strict),
        }
        print(json.dumps(line), flush=True)
    dist.destroy_process_group()

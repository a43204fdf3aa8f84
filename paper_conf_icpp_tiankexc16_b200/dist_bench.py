"""Multi-GPU arm of bench.py (torchrun, one rank per GPU, NCCL): BT class C
split into z-slabs, one halo-exchanged compute_rhs pass per step.

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
    from .rhs import coeffs_nas, init, kernel_info, launch_count, pack

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", str(rank)))
    torch.cuda.set_device(local)
    dist.init_process_group("nccl", rank=rank, world_size=world,
                            device_id=torch.device("cuda", local))
    init(local)
    bench, cls = args.config.split("-")
    n, dt = nasgen.CLASSES[(bench, cls)]
    inp = nasgen.make_class(bench, cls, seed=1)
    ug, fg = pack(inp.u, device="cpu"), pack(inp.forcing, device="cpu")
    s = sd.make_slab(ug, fg, n, rank, world, device=f"cuda:{local}")
    c = coeffs_nas(n, n, n, dt)
    comm = torch.cuda.Stream()
    compute = torch.cuda.current_stream()

    def step():
        sd.rhs_sharded(s, c, comm_stream=comm, strict=args.strict)

    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize()
    dist.barrier()
    l0 = launch_count()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(compute)
    for _ in range(args.steps):
        step()
    e1.record(compute)
    torch.cuda.synchronize()
    dist.barrier()
    ms = torch.tensor([e0.elapsed_time(e1)], device="cuda")
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    launches = torch.tensor([launch_count() - l0], device="cuda", dtype=torch.int64)
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
        step()
        hr.copy_(s.rhs, non_blocking=True)
    t1.record(compute)
    torch.cuda.synchronize()
    dist.barrier()
    ems = torch.tensor([t0.elapsed_time(t1) / args.e2e_steps], device="cuda")
    dist.all_reduce(ems, op=dist.ReduceOp.MAX)

    if rank == 0:
        line = {
            "metric": "rhs grid-points/s", "value": value, "unit": "Gpt/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": nasgen.config_name(bench, cls), "grid": [n, n, n],
                       "points": pts, "parallelism": f"z-slab x{world}, 2-plane NCCL halo",
                       "variant": "strict" if args.strict else "production",
                       "l2": "per-rank slabs; inputs > L2 at C/1-2, no flush"},
            "hbm_gbs": 120 * pts / (ms_per_step * 1e-3) / 1e9,
            "e2e": {"value": pts / (ems.item() * 1e-3) / 1e9, "unit": "Gpt/s",
                    "h2d_bytes_per_step": int((hu.numel() + hf.numel()) * 8),
                    "d2h_bytes_per_step": int(hr.numel() * 8), "note": "rank 0 slab bytes"},
            "gpu_launches": int(launches.item()),
            "kernel": kernel_info(args.strict),
        }
        print(json.dumps(line), flush=True)
    dist.destroy_process_group()

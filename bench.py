#!/usr/bin/env python
"""Benchmark: one NAS compute_rhs pass per step on B200 (BASELINE.json metric
"rhs grid-points/s and achieved HBM GB/s (% of B200 peak) at 1/2/4/8 GPUs").

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config BT-C]
  torchrun --nproc-per-node N bench.py --gpus N ...   (z-slab decomposition)
  python bench.py --impl reference ...                (CPU oracle arm)

Prints ONE JSON line on rank 0.  Workload at N=1: BT compute_rhs class C
162^3 fp64 (BASELINE.json configs[4], the class the north_star's ">= 70 % of
HBM on 1 GPU" target names).  Inputs (u 176 MB, forcing 176 MB, rhs 176 MB)
are larger than the 126 MB L2, so no L2 flush is needed between steps.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import tempfile
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

BYTES_PER_POINT = 120  # read u 40 + forcing 40, write rhs 40 (fp64, 5 comps)
FLOPS_PER_POINT = 430  # algorithmic fp64 flops (+1 reciprocal), DESIGN.md §6


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="BT-C", help="BENCH-CLASS, e.g. BT-C, SP-B")
    ap.add_argument("--grid", default=None,
                    help="nx,ny,nz override (experiments only; dt of --config)")
    ap.add_argument("--strict", action="store_true", help="time the STRICT variant")
    ap.add_argument("--dist", action="store_true",
                    help="use the z-slab/NCCL path even on one rank (testing)")
    ap.add_argument("--e2e-steps", type=int, default=20)
    ap.add_argument("--e2e-chunks", type=int, default=8,
                    help="k-chunks of the pipelined H2D / compute / D2H e2e path")
    ap.add_argument("--workload", default="rhs", choices=["rhs", "rhs_aux", "rhs_norm", "rhs_aux_norm", "seismic_dz",
                                             "bt_step"],
                    help="rhs: the headline compute_rhs pass; rhs_aux: the same pass also "
                         "writing the 6 step-0 fields (SURVEY §8(f) f1); seismic_dz: the "
                         "PAPER.md Fig. 8 loop (f4) on --seismic-n^3")
    ap.add_argument("--seismic-n", type=int, default=256)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-other-configs", action="store_true",
                    help="skip the rotating-buffer SP-B / BT-A / SP-W lines")
    ap.add_argument("--halo", default="peer", choices=["peer", "nccl"],
                    help="N>1: peer = halo fused into the kernel (loads from the neighbours' "
                         "slabs over NVLink, SURVEY f2); nccl = NCCL send/recv exchange "
                         "overlapped with the interior planes (SURVEY §8(e))")
    ap.add_argument("--graph", type=int, default=-1, metavar="G",
                    help="capture G passes into one CUDA graph and replay it K/G times (the "
                         "per-launch gap becomes a graph-internal one); default: 0 at N=1 "
                         "(back-to-back graph replays raise the power draw and the cap takes "
                         "it back in clock), 20 for the fused-halo multi-GPU path (per-rank "
                         "passes of 10-20 us, where the launch gap is 10%%)")
    ap.add_argument("--e2e-serial", action="store_true",
                    help="e2e steps without SAFARA_FLAG_PIPELINE (each step's H2D waits for "
                         "the previous step's D2H tail)")
    ap.add_argument("--e2e-canonical", action="store_true",
                    help="e2e through safara_rhs_host on the canonical pitched layout "
                         "(default: the unpadded sy = nx layout via safara_rhs_host_ex when nx is even)")
    ap.add_argument("--slab-sim", type=int, default=0, metavar="P",
                    help="one GPU: time the middle rank's fused-halo pass of a P-way "
                         "z-split (neighbour slabs resident on the same GPU) next to the "
                         "full-grid pass, and print the projected strong-scaling efficiency")
    ap.add_argument("--launch-events", action="store_true",
                    help="record an event after every launch (diagnostic; an event between "
                         "launches also serialises programmatic dependent launch)")
    ap.add_argument("--soak-s", type=float, default=1.0,
                    help="untimed passes before the timed region so the clock sampler "
                         "sees the GPU under load")
    return ap.parse_args()


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as fh:
            d = json.load(fh)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


def fp64_peak():
    """Measured DFMA peak (TFLOP/s) from the committed microbenchmark
    (tools/micro/fp64_peak.cu -> profiles/fp64_micro_r01.txt), else the
    nominal 148 SMs x 64 FP64 FMA/clk x 2 x 1.965 GHz."""
    import re
    p = os.path.join(ROOT, "profiles", "fp64_micro_r01.txt")
    if os.path.exists(p):
        vals = [float(m) for m in re.findall(r"DFMA throughput: .*?: ([0-9.]+) TFLOP/s",
                                             open(p).read())]
        if vals:
            return max(vals), "measured (profiles/fp64_micro_r01.txt, DFMA microbenchmark)"
    return 148 * 64 * 2 * 1.965e9 / 1e12, "nominal"


def ncu_entry(config_key):
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(p):
        return {}
    with open(p) as fh:
        return json.load(fh).get(config_key, {})


def ncu_traffic(config_key):
    """dram bytes per launch from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(p):
        return None
    with open(p) as fh:
        d = json.load(fh)
    e = d.get(config_key)
    return None if e is None else e.get("dram_bytes_per_launch")


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 100 ms."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.proc = None
        self.f = None

    def start(self):
        try:
            self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=self.f, stderr=subprocess.DEVNULL)
        except (OSError, FileNotFoundError):
            self.proc = None
        self.t0 = time.time()

    def mark(self):
        return time.time()

    def stop(self):
        rows = []
        if self.proc is not None:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
            self.f.flush()
            with open(self.f.name) as fh:
                for line in fh:
                    parts = [x.strip() for x in line.split(",")]
                    if len(parts) >= 9:
                        rows.append(parts)
            os.unlink(self.f.name)
        return rows

    @staticmethod
    def summarise(rows):
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        pw = [float(r[3]) for r in rows if r[3].replace(".", "").isdigit()]
        loaded = [s for s, p in zip(sm, pw) if p > 250.0] or sm
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            for n, v in zip(names, r[5:9]):
                if v.lower() == "active":
                    reasons.add(n)
        loaded.sort()
        return {"sm_mhz": loaded[len(loaded) // 2] if loaded else None,
                "sm_max_mhz": max(mx) if mx else None,
                "samples": len(rows), "samples_under_load": len(loaded),
                "power_w_max": max(pw) if pw else None,
                "reasons": sorted(reasons)}


class NvmlEnergy:
    """NVML total-energy counter (mJ) of one GPU; None when NVML is absent."""

    def __init__(self, gpu_index):
        self.h = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(gpu_index)
        except Exception:
            self.h = None

    def mj(self):
        if self.h is None:
            return None
        try:
            return self.nv.nvmlDeviceGetTotalEnergyConsumption(self.h)
        except Exception:
            return None


def power_summary(e0, e1, secs, passes, clocks, frac):
    """Board energy per pass over the untimed soak that precedes the timed
    region (same workload, back to back): the 1 kW cap binds, so joules per
    pass -- not cycles -- set the pass time.  `frac_at_sm_max`
    is a labelled what-if: the roofline fraction scaled by sm_max / sm_mhz,
    i.e. the same cycles at the unthrottled clock; it is not a measurement."""
    out = {"soak_s": round(secs, 3), "soak_passes": passes}
    if e0 is not None and e1 is not None and passes > 0 and secs > 0:
        out["w_mean"] = round((e1 - e0) / secs / 1e3, 1)
        out["mj_per_pass"] = round((e1 - e0) / passes, 3)
    sm, smx = clocks.get("sm_mhz"), clocks.get("sm_max_mhz")
    if sm and smx:
        out["frac_at_sm_max"] = round(frac * smx / sm, 4)
    return out


def cpu_oracle_time(inp, max_seconds=12.0, threads=None, min_passes=1):
    """Time the oracle as it stands on the host cores (full passes)."""
    import oracle
    threads = threads or os.cpu_count() or 1
    oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=threads)  # build + warm
    n, t0 = 0, time.perf_counter()
    while True:
        oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=threads)
        n += 1
        el = time.perf_counter() - t0
        if (el >= max_seconds and n >= min_passes) or n >= 50:
            break
    pts = inp.nx * inp.ny * inp.nz
    return {"value": pts * n / el / 1e9, "unit": "Gpt/s", "cores": threads, "kind": "oracle",
            "sample": f"{n} full {inp.nx}x{inp.ny}x{inp.nz} passes (plain C, -O2, "
                      f"-ffp-contract=off, OpenMP over k) in {el:.2f} s"}


def cpu_baseline(inp):
    """The oracle on all host cores (the reported baseline) and on ONE core
    (GPU vs one core), each a bounded sample of full passes."""
    full = cpu_oracle_time(inp, max_seconds=9.0)
    one = cpu_oracle_time(inp, max_seconds=6.0, threads=1)
    full["single_thread"] = {k: one[k] for k in ("value", "unit", "cores", "sample")}
    try:
        model = [l.split(":", 1)[1].strip() for l in open("/proc/cpuinfo")
                 if l.startswith("model name")][0]
    except (OSError, IndexError):
        model = "unknown"
    full["cpu"] = model
    return full


def other_configs(args, sr, torch, stream):
    """BASELINE.json's other configs, timed the same way but with ROTATING
    input sets whose total exceeds 2x the 126 MB L2, so each
    pass reads its inputs from HBM: these small grids are L2/launch-bound
    and reported as such (not the headline)."""
    import nasgen
    out = []
    l2 = 126e6
    for bench, cls in (("SP", "B"), ("BT", "A"), ("SP", "W")):
        n, dt = nasgen.CLASSES[(bench, cls)]
        inp = nasgen.make_class(bench, cls, seed=1)
        c = sr.coeffs_nas(n, n, n, dt)
        du, df = sr.pack(inp.u), sr.pack(inp.forcing)
        set_bytes = 3 * du.numel() * 8
        nsets = max(2, int(2 * l2 // set_bytes) + 1)
        sets = [(du.clone(), df.clone(), torch.empty_like(du)) for _ in range(nsets)]
        del du, df
        for k in range(3 * nsets):
            u, f, r = sets[k % nsets]
            sr.rhs(u, f, r, n, c, stream=stream)
        steps = max(args.steps, 10 * nsets)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for k in range(steps):
            u, f, r = sets[k % nsets]
            sr.rhs(u, f, r, n, c, stream=stream)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / steps
        pts = n ** 3
        out.append({"workload": nasgen.config_name(bench, cls), "value": pts / (ms * 1e-3) / 1e9,
                    "unit": "Gpt/s", "us_per_pass": ms * 1e3,
                    "hbm_frac": BYTES_PER_POINT * pts / (ms * 1e-3) / 1e9 / measured_peaks()[0],
                    "l2": f"rotating {nsets} input sets of {set_bytes / 1e6:.1f} MB "
                          f"({nsets * set_bytes / 1e6:.0f} MB > 2x L2)",
                    "bound": "L2/launch-bound (small grid), effective throughput"})
        del sets
    return out


def config_of(args):
    import nasgen
    bench, cls = args.config.split("-")
    n, dt = nasgen.CLASSES[(bench, cls)]
    return bench, cls, n, dt


def grid_of(args, n):
    if args.grid:
        nx, ny, nz = (int(v) for v in args.grid.split(","))
        return nx, ny, nz
    return n, n, n


def run_reference(args):
    """CPU oracle arm (rank 0 only)."""
    import nasgen
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    bench, cls, n, dt = config_of(args)
    inp = nasgen.make_class(bench, cls, seed=1)
    import oracle
    threads = os.cpu_count() or 1
    for _ in range(max(args.warmup, 0)):
        oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=threads)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt, threads=threads)
        times.append(time.perf_counter() - t0)
    tot = sum(times)
    pts = n ** 3
    value = pts * args.steps / tot / 1e9
    line = {
        "impl": "reference", "metric": "rhs grid-points/s", "value": value, "unit": "Gpt/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": tot / args.steps * 1e3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": nasgen.config_name(bench, cls), "grid": [n, n, n],
                   "points": pts, "l2": "host"},
        "cpu_baseline": {"value": value, "unit": "Gpt/s", "cores": threads, "kind": "oracle",
                         "sample": f"{args.steps} full {n}^3 passes of the plain-C oracle",
                         "single_thread": {k: v for k, v in cpu_oracle_time(
                             inp, max_seconds=6.0, threads=1).items()
                             if k in ("value", "unit", "cores", "sample")}},
        "e2e": {"value": value, "unit": "Gpt/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def run_single(args):
    import torch

    import nasgen
    import paper_conf_icpp_tiankexc16_b200 as sr

    torch.cuda.set_device(0)
    sr.init(0)
    bench, cls, n, dt = config_of(args)
    nx, ny, nz = grid_of(args, n)
    if args.grid:
        inp = nasgen.make_inputs(nx, ny, nz, seed=1, dt=dt, bench=bench, cls=cls)
    else:
        inp = nasgen.make_class(bench, cls, seed=1)
    c = sr.coeffs_nas(nx, ny, nz, dt)
    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    dr = torch.empty_like(du)
    stream = torch.cuda.current_stream()
    pts = nx * ny * nz
    bytes_per_point = BYTES_PER_POINT
    if args.workload == "rhs_aux":
        da = sr.empty_aux(nx, ny, nz, sr.SAFARA_AUX_BT)
        bytes_per_point += 8 * sr.SAFARA_AUX_BT

        def step(st=None):
            sr.rhs_aux(du, df, dr, da, nx, c, strict=args.strict, stream=st or stream)
    elif args.workload in ("rhs_norm", "rhs_aux_norm"):
        # f1: rhs_norm accumulated in the store epilogue (+ the aux fields)
        da = sr.empty_aux(nx, ny, nz, sr.SAFARA_AUX_BT) if args.workload == "rhs_aux_norm" else None
        if da is not None:
            bytes_per_point += 8 * sr.SAFARA_AUX_BT
        rms_out = torch.empty(5, dtype=torch.float64, device="cuda")

        def step(st=None):
            sr.rhs_fused(du, df, dr, nx, c, aux=da, rms=rms_out, strict=args.strict,
                         stream=st or stream)
    else:
        def step(st=None):
            sr.rhs(du, df, dr, nx, c, strict=args.strict, stream=st or stream)

    graph, replays = None, 0
    if args.graph > 0:
        G = args.graph
        args.steps = max(G, (args.steps // G) * G)
        replays = args.steps // G
        for _ in range(3):
            step()
        torch.cuda.synchronize()
        graph = torch.cuda.CUDAGraph()
        g0 = sr.launch_count()
        with torch.cuda.graph(graph):
            cs = torch.cuda.current_stream()
            for _ in range(G):
                step(cs)
        per_graph_launches = sr.launch_count() - g0
        torch.cuda.synchronize()

        def step(st=None):  # noqa: F811 -- one replay = G passes
            graph.replay()

    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize()

    sampler = ClockSampler(0)
    sampler.start()
    nvml = NvmlEnergy(0)
    e_soak0, t_soak0, n_soak = nvml.mj(), time.time(), 0
    t_end = time.time() + args.soak_s
    while time.time() < t_end:
        for _ in range(50):
            step()
        n_soak += 50 * (G if graph is not None else 1)
        torch.cuda.synchronize()
    e_soak1, t_soak1 = nvml.mj(), time.time()

    # timed region: K steps, per-launch events on the launching stream
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]
    l0 = sr.launch_count()
    torch.cuda.synchronize()
    # window events (stream launches only): 5 equal windows of the K passes,
    # for the min / median per-pass spread SURVEY §8(d) asks about
    nwin = 5 if (graph is None and not args.launch_events and args.steps >= 10) else 0
    wev = {args.steps * w // nwin: torch.cuda.Event(enable_timing=True)
           for w in range(1, nwin)} if nwin else {}
    ev[0].record(stream)
    for k in range(replays if graph is not None else args.steps):
        step()
        if args.launch_events and graph is None:
            ev[k + 1].record(stream)
        elif k + 1 in wev:
            wev[k + 1].record(stream)
    if not args.launch_events or graph is not None:
        ev[-1].record(stream)
    torch.cuda.synchronize()
    windows = None
    if nwin:
        bounds = [0] + sorted(wev) + [args.steps]
        evs = [ev[0]] + [wev[b] for b in sorted(wev)] + [ev[-1]]
        wms = sorted(evs[w].elapsed_time(evs[w + 1]) * 1e3 / (bounds[w + 1] - bounds[w])
                     for w in range(nwin))
        windows = {"n": nwin, "us_per_pass_min": round(wms[0], 2),
                   "us_per_pass_median": round(wms[nwin // 2], 2),
                   "us_per_pass_max": round(wms[-1], 2)}
    launches = sr.launch_count() - l0 + (per_graph_launches * replays if graph is not None else 0)
    total_ms = ev[0].elapsed_time(ev[-1])
    # one launch per step: the average launch duration is the step time
    per = ([ev[k].elapsed_time(ev[k + 1]) for k in range(args.steps)]
           if args.launch_events and graph is None else [total_ms / args.steps])
    rows = sampler.stop()
    clocks = ClockSampler.summarise(rows)

    ms_per_step = total_ms / args.steps
    value = pts / (ms_per_step * 1e-3) / 1e9
    kern_ms = sum(per) / len(per)
    achieved = bytes_per_point * pts / (kern_ms * 1e-3) / 1e9
    peak, peak_kind = measured_peaks()
    key = f"{bench}-{cls}"
    traffic = ncu_traffic(key)
    fpk, fpk_kind = fp64_peak()
    ncu_e = ncu_entry(key)
    fp64_tf = FLOPS_PER_POINT * pts / (kern_ms * 1e-3) / 1e12

    # e2e: host (pinned) buffers through the C ABI, H2D + pass + D2H per step
    e2e_ms, nbytes = float("nan"), 0
    e2e_layout = None
    if args.e2e_steps > 0 and args.workload == "rhs":
        import numpy as np
        if nx % 2 == 0 and not args.e2e_canonical:
            # the NAS-native unpadded layout (sy = nx) through safara_rhs_host_ex:
            # 3.6 % fewer PCIe bytes than the canonical pitch at class C
            def host(a):
                t = torch.empty((nz, 5, ny, nx), dtype=torch.float64).pin_memory()
                t.copy_(torch.from_numpy(np.ascontiguousarray(a)).permute(0, 3, 1, 2))
                return t
            hu, hf = host(inp.u), host(inp.forcing)
            hr = torch.empty(hu.shape, dtype=torch.float64).pin_memory()
            eu, ef, er = (torch.empty(hu.shape, dtype=torch.float64, device="cuda") for _ in range(3))
            dd = sr.Dims(nx, ny, nz, nx, ny * nx, 5 * ny * nx)
            e2e_layout = "unpadded sy = nx (safara_rhs_host_ex)"

            def e2e_step():
                sr.rhs_host_ex(hu, hf, hr, eu, ef, er, dd, c, strict=args.strict,
                               nchunks=args.e2e_chunks, stream=stream,
                               pipeline=not args.e2e_serial)
        else:
            hu, hf = sr.pack(inp.u, pin=True), sr.pack(inp.forcing, pin=True)
            hr = torch.empty(hu.shape, dtype=torch.float64).pin_memory()
            e2e_layout = f"canonical pitch sy = {sr.pitch(nx)} (safara_rhs_host)"

            def e2e_step():
                sr.rhs_host(hu, hf, hr, du, df, dr, nx, c, strict=args.strict,
                            nchunks=args.e2e_chunks, stream=stream,
                            pipeline=not args.e2e_serial)
        for _ in range(2):
            e2e_step()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.e2e_steps):
            e2e_step()
        e1.record(stream)
        torch.cuda.synchronize()
        e2e_ms = e0.elapsed_time(e1) / args.e2e_steps
        nbytes = hu.numel() * 8

    line = {
        "metric": "rhs grid-points/s", "value": value, "unit": "Gpt/s",
        "n_gpus": 1, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": nasgen.config_name(bench, cls) if not args.grid else
                   f"{bench} compute_rhs {nx}x{ny}x{nz} fp64 (experiment grid)", "grid": [nx, ny, nz],
                   "points": pts, "variant": "strict" if args.strict else "production",
                   "l2": "inputs 3x176 MB > 126 MB L2, no flush", "parallelism": "single",
                   "launch": (f"CUDA graph of {args.graph} passes, replayed {replays}x"
                              if graph is not None else "one stream launch per pass")},
        "hbm_gbs": achieved,
        "windows": windows,
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "peak_kind": peak_kind, "traffic": traffic,
                     "bytes_per_point": bytes_per_point, "kernel_ms": kern_ms,
                     "frac_of_8000": achieved / 8000.0},
        "roofline_fp64": {"bound": "fp64", "achieved": fp64_tf, "peak": fpk,
                          "unit": "TFLOP/s", "frac": fp64_tf / fpk, "peak_kind": fpk_kind,
                          "flops_per_point": FLOPS_PER_POINT,
                          "ncu_fp64_pipe_active_pct": ncu_e.get("fp64_pipe_active_pct"),
                          "note": "algorithmic flops (430/pt); the FP64 pipe is the "
                                  "near-binding second roofline (DESIGN.md §5)"},
        "clocks": clocks,
        "power": power_summary(e_soak0, e_soak1, t_soak1 - t_soak0, n_soak, clocks,
                               achieved / peak),
        "e2e": {"value": pts / (e2e_ms * 1e-3) / 1e9, "unit": "Gpt/s",
                "h2d_bytes_per_step": 2 * nbytes, "d2h_bytes_per_step": nbytes,
                "ms_per_step": e2e_ms, "host_layout": e2e_layout,
                "pipelined": bool(args.e2e_steps > 0 and not args.e2e_serial)},
        "gpu_launches": launches,
        "kernel": sr.kernel_info(args.strict),
    }
    if not args.no_other_configs and args.workload == "rhs" and not args.grid:
        line["other_configs"] = other_configs(args, sr, torch, stream)
    if not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(inp)
    print(json.dumps(line), flush=True)


def run_bt_step(args):
    """one whole NPB BT time step per step (safara_bt_step:
    compute_rhs with the aux fields, x/y/z block-tridiagonal line solves, add;
    5 launches) at the class of --config (BT-C by default), from NPB's
    initialize with exact_rhs forcing; reported in grid-points/s of steps.
    The line solves are a plain one-thread-per-line kernel (not the tuned
    path); this line measures the whole step, not a roofline claim."""
    import torch

    import nasgen
    import paper_conf_icpp_tiankexc16_b200 as sr

    torch.cuda.set_device(0)
    sr.init(0)
    bench, cls, n, dt = config_of(args)
    u0 = nasgen.nas_initialize(n, n, n)
    f = nasgen.exact_rhs(n, n, n, dt)
    st = sr.BtState(sr.pack(u0), sr.pack(f), n, dt)
    stream = torch.cuda.current_stream()
    for _ in range(max(args.warmup, 3)):
        st.step(strict=args.strict)
    torch.cuda.synchronize()
    sampler = ClockSampler(0)
    sampler.start()
    l0 = sr.launch_count()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        st.step(strict=args.strict)
    e1.record(stream)
    torch.cuda.synchronize()
    clocks = ClockSampler.summarise(sampler.stop())
    ms = e0.elapsed_time(e1) / args.steps
    pts = n ** 3
    print(json.dumps({
        "metric": "BT time steps x grid-points/s", "value": pts / (ms * 1e-3) / 1e9,
        "unit": "Gpt/s", "n_gpus": 1, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": ms, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "f64", "data": "synthetic (NPB initialize + exact_rhs)",
        "config": {"workload": f"NPB BT time step class {cls} {n}^3 fp64 (f4(ii))",
                   "grid": [n, n, n], "points": pts,
                   "variant": "strict" if args.strict else "production"},
        "clocks": clocks, "gpu_launches": sr.launch_count() - l0}), flush=True)


def run_seismic(args):
    """PAPER.md Fig. 8 dz loop: 3 inputs + 1 output of
    n^3 doubles, 32 algorithmic bytes per point (HBM-bound)."""
    import numpy as np
    import torch

    import paper_conf_icpp_tiankexc16_b200 as sr

    torch.cuda.set_device(0)
    sr.init(0)
    n = args.seismic_n
    sy = sr.pitch(n)
    g = torch.Generator(device="cuda").manual_seed(1)
    vz = [torch.randn((n, n, sy), dtype=torch.float64, device="cuda", generator=g)
          for _ in range(3)]
    out = torch.zeros_like(vz[0])
    stream = torch.cuda.current_stream()
    pts = (n - 1) ** 3  # written points
    for _ in range(max(args.warmup, 3)):
        sr.seismic_dz(*vz, out, 0.01, n, stream=stream)
    sampler = ClockSampler(0)
    sampler.start()
    t_end = time.time() + args.soak_s
    while time.time() < t_end:
        for _ in range(20):
            sr.seismic_dz(*vz, out, 0.01, n, stream=stream)
        torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]
    l0 = sr.launch_count()
    torch.cuda.synchronize()
    ev[0].record(stream)
    for k in range(args.steps):
        sr.seismic_dz(*vz, out, 0.01, n, stream=stream)
        ev[k + 1].record(stream)
    torch.cuda.synchronize()
    per = [ev[k].elapsed_time(ev[k + 1]) for k in range(args.steps)]
    clocks = ClockSampler.summarise(sampler.stop())
    ms = ev[0].elapsed_time(ev[-1]) / args.steps
    kern_ms = float(np.mean(per))
    peak, peak_kind = measured_peaks()
    achieved = 32 * pts / (kern_ms * 1e-3) / 1e9
    print(json.dumps({
        "metric": "seismic dz grid-points/s", "value": pts / (ms * 1e-3) / 1e9, "unit": "Gpt/s",
        "n_gpus": 1, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic",
        "config": {"workload": f"355.seismic dz loop (PAPER.md Fig. 8) {n}^3 fp64",
                   "grid": [n, n, n], "points": pts,
                   "l2": f"4 x {n * n * sy * 8 / 1e6:.0f} MB > 126 MB L2, no flush"},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "peak_kind": peak_kind, "traffic": None,
                     "bytes_per_point": 32, "kernel_ms": kern_ms},
        "clocks": clocks, "gpu_launches": sr.launch_count() - l0}), flush=True)


def run_slab_sim(args):
    """Per-rank pass time of a P-way z-split, measured on one GPU: the middle
    rank's safara_rhs_peer launch (its neighbours' slabs live on the same GPU,
    epoch 0), K passes between two events, against the full-grid pass timed
    the same way.  Projects T1 / (P * Tp); NVLink peer loads (2 x 2 own-column
    planes per pass) and cross-GPU flag waits are not included."""
    import torch

    import nasgen
    import paper_conf_icpp_tiankexc16_b200 as sr
    from paper_conf_icpp_tiankexc16_b200 import dist as sd

    torch.cuda.set_device(0)
    sr.init(0)
    bench, cls, n, dt = config_of(args)
    inp = nasgen.make_class(bench, cls, seed=1)
    c = sr.coeffs_nas(n, n, n, dt)
    stream = torch.cuda.current_stream()

    def timed(fn):
        for _ in range(max(args.warmup, 3)):
            fn()
        torch.cuda.synchronize()
        if args.graph > 0:
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                for _ in range(args.graph):
                    fn(torch.cuda.current_stream())
            reps = max(1, args.steps // args.graph)
            g.replay()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            for _ in range(reps):
                g.replay()
            e1.record(stream)
            torch.cuda.synchronize()
            return e0.elapsed_time(e1) / (reps * args.graph)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.steps):
            fn()
        e1.record(stream)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / args.steps

    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    dr = torch.empty_like(du)
    t1 = timed(lambda st=None: sr.rhs(du, df, dr, n, c, stream=st or stream))
    del du, df, dr
    p = args.slab_sim
    ug, fg = sr.pack(inp.u, device="cpu"), sr.pack(inp.forcing, device="cpu")
    r = p // 2
    nb = sd.neighbours(n, p, r)
    slabs = {q: sd.make_slab(ug, fg, n, q, p, device="cuda") for q in (nb["lo"], r, nb["hi"])
             if q is not None}
    s = slabs[r]
    pr = sd.peer_struct(nb, slabs[nb["lo"]].u.data_ptr() if nb["lo"] is not None else None,
                        slabs[nb["hi"]].u.data_ptr() if nb["hi"] is not None else None,
                        None, None, None, 0)
    tp = timed(lambda st=None: sr.rhs_peer(s.u, s.forcing, s.rhs, n, n, s.k0, pr, c,
                                           stream=st or stream))
    print(json.dumps({"slab_sim": p, "rank": r, "planes": s.nzl, "config": f"{bench}-{cls}",
                      "t1_ms": t1, "tp_ms": tp, "projected_efficiency": t1 / (p * tp),
                      "steps": args.steps, "graph": args.graph}), flush=True)


def main():
    args = parse()
    if args.graph < 0:
        multi = int(os.environ.get("WORLD_SIZE", "1")) > 1 or args.gpus > 1
        args.graph = 20 if multi and args.halo == "peer" else 0
    if args.slab_sim:
        run_slab_sim(args)
        return
    if args.workload == "bt_step" and args.impl != "reference":
        run_bt_step(args)
        return
    if args.workload == "seismic_dz" and args.impl != "reference":
        run_seismic(args)
        return
    if args.impl == "reference":
        run_reference(args)
        return
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world > 1 or args.gpus > 1 or args.dist:
        from paper_conf_icpp_tiankexc16_b200 import dist_bench
        dist_bench.run(args)
    else:
        run_single(args)


if __name__ == "__main__":
    main()

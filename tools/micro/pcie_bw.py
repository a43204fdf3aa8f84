"""PCIe copy-engine bandwidth on the box (pinned host memory): one H2D stream,
two H2D streams, H2D || D2H -- what bounds the e2e host path."""
import torch

N = 340 * 2**20 // 8
h = torch.empty(N, dtype=torch.float64).pin_memory()
h2 = torch.empty(N, dtype=torch.float64).pin_memory()
d = torch.empty(N, dtype=torch.float64, device="cuda")
d2 = torch.empty(N, dtype=torch.float64, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def timed(fn, reps=5):
    best = 1e9
    for _ in range(reps):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        for s in (s1, s2):
            torch.cuda.current_stream().wait_stream(s)
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best


def h2d1():
    with torch.cuda.stream(s1):
        d.copy_(h, non_blocking=True)


def h2d2():
    with torch.cuda.stream(s1):
        d[:N // 2].copy_(h[:N // 2], non_blocking=True)
    with torch.cuda.stream(s2):
        d[N // 2:].copy_(h[N // 2:], non_blocking=True)


def both():
    with torch.cuda.stream(s1):
        d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2):
        h2[:N // 2].copy_(d2[:N // 2], non_blocking=True)


gb = N * 8 / 1e9
t = timed(h2d1); print(f"H2D 340 MB, 1 stream: {t:.2f} ms  {gb / t * 1e3:.1f} GB/s")
t = timed(h2d2); print(f"H2D 340 MB, 2 streams: {t:.2f} ms  {gb / t * 1e3:.1f} GB/s")
t = timed(both); print(f"H2D 340 MB || D2H 170 MB: {t:.2f} ms  H2D {gb / t * 1e3:.1f} GB/s")

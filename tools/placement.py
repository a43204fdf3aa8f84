"""Does the relative placement of u / forcing / rhs in device memory change the
BT-C pass time?  One process, one pool allocation; the three fields are views
at configurable byte offsets (multiples of 2 MiB plus a shift); each layout is
timed (1 s soak at the power cap, then 200 passes, CUDA events) in rounds.

  python tools/placement.py [rounds]
"""
import sys
import time

import torch

sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__file__)))
import nasgen  # noqa: E402
import paper_conf_icpp_tiankexc16_b200 as sr  # noqa: E402

rounds = int(sys.argv[1]) if len(sys.argv) > 1 else 2
sr.init(0)
inp = nasgen.make_class("BT", "C", seed=1)
du0, df0 = sr.pack(inp.u), sr.pack(inp.forcing)
n = du0.numel()
MB2 = 2 * 2**20 // 8  # doubles per 2 MiB
pool = torch.empty(3 * n + 64 * MB2, dtype=torch.float64, device="cuda")
c = sr.coeffs_nas(162, 162, 162, inp.dt)
shape = du0.shape
# (name, u offset, f offset, r offset) in doubles from the pool start
lay = {
    "packed": (0, n, 2 * n),
    "gap1MiB": (0, n + MB2 // 2, 2 * n + MB2),
    "gap2MiB": (0, n + MB2, 2 * n + 2 * MB2),
    "gap6MiB": (0, n + 3 * MB2, 2 * n + 6 * MB2),
    "gap32MiB": (0, n + 16 * MB2, 2 * n + 32 * MB2),
    "rfu": (2 * n + 4 * MB2, n + 2 * MB2, 0),
}
views = {}
for name, (ou, of, orr) in lay.items():
    views[name] = tuple(pool[o:o + n].view(shape) for o in (ou, of, orr))


def time_layout(du, df, dr, k=200):
    du.copy_(du0)
    df.copy_(df0)
    for _ in range(20):
        sr.rhs(du, df, dr, 162, c)
    torch.cuda.synchronize()
    t = time.time()
    while time.time() - t < 1.0:
        for _ in range(50):
            sr.rhs(du, df, dr, 162, c)
        torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(k):
        sr.rhs(du, df, dr, 162, c)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / k


print("pool base 0x%x" % pool.data_ptr())
for r in range(rounds):
    for name, (du, df, dr) in views.items():
        print(f"round {r} {name:9s} {time_layout(du, df, dr):8.2f} us", flush=True)

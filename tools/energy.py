"""Energy per compute_rhs pass on the B200 (the bench is power-capped at 1 kW).

  python tools/energy.py SPEC ...     (on the GPU box)

SPEC = LIB[+ENV=V...] as in tools/ab.py (LIB 'default' or a name under
ablibs/), or the pseudo-specs 'idle' (sleep) and 'copy' (a torch copy moving
the pass's algorithmic bytes: read 353 MB, write 176 MB).  Each spec runs in
its own process: BT class C, ~2 s of back-to-back passes after a 1 s soak;
NVML's total-energy counter (mJ) and CUDA events bracket the timed passes.
Prints one JSON line per spec: us/pass, mJ/pass, mean W, median SM MHz.
"""
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ABLIBS = os.path.join(ROOT, "ablibs")

CHILD = r"""
import json, os, sys, time, threading
sys.path.insert(0, os.environ['ROOT'])
import torch, pynvml
pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(0)
spec = os.environ['SPEC']
clk = []
stop = False
def sampler():
    while not stop:
        clk.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)); time.sleep(0.05)
if spec == 'idle':
    torch.zeros(1, device='cuda'); torch.cuda.synchronize()
    e0 = pynvml.nvmlDeviceGetTotalEnergyConsumption(h); t0 = time.time(); time.sleep(2.0)
    e1 = pynvml.nvmlDeviceGetTotalEnergyConsumption(h); t1 = time.time()
    print(json.dumps({'spec': spec, 'W': (e1 - e0) / (t1 - t0) / 1e3}))
    sys.exit(0)
if spec == 'copy':
    a = torch.empty(2 * 5 * 162 * 162 * 168, dtype=torch.float64, device='cuda')
    b = torch.empty(5 * 162 * 162 * 168, dtype=torch.float64, device='cuda')
    def one():
        torch.add(a[:b.numel()], a[b.numel():], out=b)
else:
    import nasgen, paper_conf_icpp_tiankexc16_b200 as sr
    sr.init(0)
    inp = nasgen.make_class('BT', 'C')
    du, df = sr.pack(inp.u), sr.pack(inp.forcing)
    dr = torch.empty_like(du)
    co = sr.coeffs_nas(162, 162, 162, inp.dt)
    def one():
        sr.rhs(du, df, dr, 162, co)
for _ in range(20): one()
torch.cuda.synchronize()
t0 = time.time()
while time.time() - t0 < 1.0: one()
torch.cuda.synchronize()
n = 0; ev0 = torch.cuda.Event(enable_timing=True); ev1 = torch.cuda.Event(enable_timing=True)
th = threading.Thread(target=sampler); th.start()
# ~2 s: measure one batch first to size it
ev0.record()
for _ in range(50): one()
ev1.record(); torch.cuda.synchronize()
per = ev0.elapsed_time(ev1) / 50
K = max(100, int(2000 / per))
e0 = pynvml.nvmlDeviceGetTotalEnergyConsumption(h)
ev0.record()
for _ in range(K): one()
ev1.record(); torch.cuda.synchronize()
e1 = pynvml.nvmlDeviceGetTotalEnergyConsumption(h)
stop = True; th.join()
ms = ev0.elapsed_time(ev1)
clk.sort()
print(json.dumps({'spec': spec, 'us': round(ms * 1e3 / K, 2), 'mJ': round((e1 - e0) / K, 3),
                  'W': round((e1 - e0) / ms, 1), 'sm_mhz': clk[len(clk) // 2] if clk else None,
                  'K': K}))
"""


def main(specs, reps=1):
    for rep in range(reps):
        for spec in specs:
            lib, *envs = spec.split("+")
            env = dict(os.environ, ROOT=ROOT, SPEC=lib if lib in ("idle", "copy") else spec)
            if lib not in ("default", "idle", "copy"):
                env["SAFARA_LIB"] = os.path.join(ABLIBS, lib + ".so")
            for e in envs:
                k, _, v = e.partition("=")
                env[k] = v
            r = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True,
                               text=True, timeout=300)
            out = r.stdout.strip().splitlines()
            print(out[-1] if out else json.dumps({"spec": spec, "error": r.stderr[-400:]}),
                  flush=True)
            time.sleep(1.0)


if __name__ == "__main__":
    args = sys.argv[1:]
    reps = 1
    if args and args[0].startswith("--reps="):
        reps = int(args[0].split("=")[1])
        args = args[1:]
    main(args, reps)

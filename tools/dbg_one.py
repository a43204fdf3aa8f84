"""Run one small pass (both variants) and compare with the oracle: a quick
debugging / compute-sanitizer target.  usage: python tools/dbg_one.py [n] [strict]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import nasgen
import oracle
import paper_conf_icpp_tiankexc16_b200 as sr

n = int(sys.argv[1]) if len(sys.argv) > 1 else 12
sr.init(0)
inp = nasgen.make_inputs(n, n, n, seed=1, dt=0.01)
c = sr.coeffs_nas(n, n, n, inp.dt)
du, df = sr.pack(inp.u), sr.pack(inp.forcing)
o = oracle.compute_rhs(inp.u, inp.forcing, dt=inp.dt)
for strict in (True, False):
    dr = torch.full_like(du, float("nan"))
    sr.rhs(du, df, dr, n, c, strict=strict)
    torch.cuda.synchronize()
    g = sr.unpack(dr, n)
    d = np.abs(g - o)
    print(f"n={n} strict={strict}: max|g-o|={np.nanmax(d):.3g} nan={np.isnan(g).sum()} "
          f"bitwise={np.array_equal(g, o)}")
    if not np.array_equal(g, o):
        bad = np.argwhere(~(d <= 1e-12 * np.abs(o) + 1e-14))
        print("  first bad (k,j,i,m):", bad[:8].tolist())

import os, sys
sys.path.insert(0, os.getcwd())
import torch, numpy as np, nasgen, oracle
import paper_conf_icpp_tiankexc16_b200 as sr
sr.init(0)
inp = nasgen.make_class("BT", "S", seed=1)
nz, ny, nx, _ = inp.u.shape
c = sr.coeffs_nas(nx, ny, nz, inp.dt)
du, df = sr.pack(inp.u), sr.pack(inp.forcing)
dr = torch.empty_like(du)
for strict in (False, True):
    try:
        sr.rhs(du, df, dr, nx, c, strict=strict); torch.cuda.synchronize(); print("rhs ok", strict)
    except Exception as e:
        print("rhs fail", strict, e)
from paper_conf_icpp_tiankexc16_b200 import dist as sd
s = sd.make_slab(sr.pack(inp.u, device="cpu"), sr.pack(inp.forcing, device="cpu"), nx, 0, 1, device="cuda")
for strict in (False, True):
    try:
        sr.rhs_slab(s.u, s.forcing, s.rhs, nx, nz, 0, c, strict=strict); torch.cuda.synchronize(); print("slab ok", strict)
    except Exception as e:
        print("slab fail", strict, e)
print(s.u.data_ptr() % 256, du.data_ptr() % 256)

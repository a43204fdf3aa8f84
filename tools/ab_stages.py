"""A/B the TMA ring depth (SAFARA_STAGES) of the production kernel on one box,
interleaved runs of bench.py against per-variant library builds (f3 tuner)."""
import json
import sys

from paper_conf_icpp_tiankexc16_b200.safara_tune import Variant, time_variant

variants = [Variant(12, 4, 2), Variant(12, 5, 2)]
res = {v.tag(): [] for v in variants}
for rep in range(int(sys.argv[1]) if len(sys.argv) > 1 else 3):
    for v in variants:
        res[v.tag()].append(time_variant((v.tag(), v.defines()), steps=200))
        print(json.dumps({"variant": v.tag(), "rep": rep, "kernel_us": res[v.tag()][-1]}), flush=True)
print(json.dumps({k: sorted(x for x in t if x) for k, t in res.items()}))

#!/bin/bash
# A/B of the warp-specialised kernel (SAFARA_WS=1) against the round-1 kernel
# (SAFARA_WS=0) on BT class C: interleaved bench runs, kernel-time lines only.
out=${1:-gpurun_out/ab_ws.txt}
: > "$out"
for rep in 1 2 3; do
  for ws in 0 1; do
    SAFARA_WS=$ws timeout 300 python bench.py --no-cpu-baseline --e2e-steps 1 --steps 400 --warmup 20 2>/dev/null \
      | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print('ws=$ws', round(d['ms_per_step']*1e3,2), 'us', round(d['value'],2), 'Gpt/s frac', round(d['roofline']['frac'],3), 'sm', d['clocks']['sm_mhz'])" >> "$out"
  done
done
cat "$out"

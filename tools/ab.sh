#!/bin/bash
# A/B timing of variant builds: tools/ab.sh <steps> <lib.so>[:ENV=V,...] ...
steps=$1; shift
for spec in "$@"; do
  lib=${spec%%:*}; envs=""
  [[ "$spec" == *:* ]] && envs=${spec#*:}
  line=$(env ${envs//,/ } SAFARA_LIB=$PWD/$lib timeout 300 python bench.py --steps $steps --warmup 10 --no-cpu-baseline --soak-s 0.3 --e2e-steps 1 $AB_ARGS 2>&1 | tail -1)
  python - "$spec" "$line" <<'PY'
import json, sys
spec, line = sys.argv[1], sys.argv[2]
try:
    d = json.loads(line)
    print(f"{spec:40s} {d['value']:7.2f} Gpt/s  {d['roofline']['achieved']:7.0f} GB/s  frac={d['roofline']['frac']:.3f}  kern={d["roofline"]["kernel_ms"]*1e3:.1f}us grid={d["config"]["grid"]}  sm={d['clocks'].get('sm_mhz')}")
except Exception as e:
    print(spec, "ERROR", line[-300:])
PY
done

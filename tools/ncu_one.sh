#!/bin/bash
# One `ncu --set full` capture of the production rhs kernel (launch 6 of a
# short bench run).  usage: tools/ncu_one.sh <out-name> [env assignments...]
name=$1; shift
env "$@" timeout 900 ncu --set full --import-source on --clock-control none \
  -k regex:rhs_kernel_fast -c 1 --launch-skip 5 -f -o gpurun_out/$name \
  python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-other-configs --e2e-steps 1 --soak-s 0.1 > gpurun_out/$name.log 2>&1
echo "ncu $name rc=$?"

#!/bin/bash
# interleaved bench runs of several workloads for the default library and
# ablibs/$1.so: kernel us per pass.  usage: tools/ab_workloads.sh LIB [reps]
lib=$1; reps=${2:-2}
for rep in $(seq $reps); do for w in rhs rhs_norm rhs_aux rhs_aux_norm; do for L in default $lib; do
  if [ $L = default ]; then unset SAFARA_LIB; else export SAFARA_LIB=ablibs/$L.so; fi
  timeout 200 python bench.py --workload $w --no-cpu-baseline --no-other-configs --e2e-steps 0 --steps 300 2>/dev/null \
   | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print('$L', '$w', round(d['ms_per_step']*1e3,2), d['clocks']['sm_mhz'])"
done; done; done

#!/bin/bash
# Round evidence for profiles/: ncu --set full of the production kernel (one
# launch of a short BT-C bench run), the launch list (gpu__time_duration of
# every kernel of a bench run: kernel shares of the step), and the summary.
# usage: tools/profile_round.sh rNN
r=${1:-r02}
bash tools/ncu_one.sh ncu_full_$r
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/ncu_launches_$r.csv \
  python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-other-configs --e2e-steps 1 --soak-s 0.2 \
  > gpurun_out/ncu_launches_$r.log 2>&1
echo "launch list rc=$?"

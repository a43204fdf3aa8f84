cd $GRAFT_REPO_ROOT
ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv --log-file gpurun_out/launches.csv python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 --soak-s 0 > gpurun_out/ncu_bench.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:rhs_kernel -s 5 -c 1 -o gpurun_out/prof -f python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 --soak-s 0 > gpurun_out/ncu_full.log 2>&1
python tools/ncu_summary.py gpurun_out/prof.ncu-rep > gpurun_out/ncu_full_summary.txt 2>&1
SAFARA_LIB=$PWD/ablibs/tl.so timeout 300 python bench.py --steps 50 --warmup 5 --no-cpu-baseline --e2e-steps 0 --soak-s 0.5 > gpurun_out/tl_bench.json 2>&1
cp gpurun_out/timeline.txt gpurun_out/timeline_full.txt

# Round-end validation pass run on the GPU box via gpurun (also used as the
# scratch script for experiments).
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.txt 2>&1
python __graft_entry__.py --smoke > gpurun_out/smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 python bench.py --strict --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_strict.json 2>&1
timeout 300 python bench.py --workload rhs_aux --steps 100 --no-cpu-baseline > gpurun_out/bench_aux.json 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.json 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv --log-file gpurun_out/launches.csv python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 --soak-s 0 > gpurun_out/ncu_bench.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:rhs_kernel -s 5 -c 1 -o gpurun_out/prof -f python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 --soak-s 0 > gpurun_out/ncu_full.log 2>&1
python tools/ncu_summary.py gpurun_out/prof.ncu-rep > gpurun_out/ncu_full_summary.txt 2>&1
SAFARA_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 40 --warmup 3 --e2e-steps 2 --soak-s 0.2 > gpurun_out/dist2g.json 2>&1

# One GPU round-trip: parity tests, the headline bench, the f1/f4 workloads,
# and the SAFARA variant tuner's timing leg.
set -x
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 python bench.py --workload rhs_aux --steps 100 --no-cpu-baseline > gpurun_out/bench_aux.json 2>&1
timeout 300 python bench.py --workload seismic_dz --steps 100 > gpurun_out/bench_seismic.json 2>&1
timeout 900 python -m paper_conf_icpp_tiankexc16_b200.safara_tune --time 4 --jobs 8 > gpurun_out/safara_tune.txt 2>&1

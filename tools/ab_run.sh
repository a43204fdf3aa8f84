# Scratch experiment script run on the GPU box via gpurun (edited per
# experiment; the committed version is the round-end validation pass).
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.txt 2>&1
python __graft_entry__.py --smoke > gpurun_out/smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
for cfg in "BT-C 2" "BT-C 4" "BT-C 8" "SP-B 2" "SP-B 4" "SP-B 8"; do set -- $cfg; for g in 0 20; do timeout 300 python bench.py --slab-sim $2 --config $1 --steps 400 --warmup 10 --graph $g; done; done > gpurun_out/slabsim_final.txt 2>&1
SAFARA_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 40 --warmup 3 --e2e-steps 2 --soak-s 0.2 > gpurun_out/dist2g.json 2>&1

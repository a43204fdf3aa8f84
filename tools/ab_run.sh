# Scratch experiment script run on the GPU box via gpurun (edited per
# experiment; the committed version is the round-end validation pass).
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.txt 2>&1
python __graft_entry__.py --smoke > gpurun_out/smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
SAFARA_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 40 --warmup 3 --e2e-steps 2 --soak-s 0.2 > gpurun_out/dist2g.json 2>&1
SAFARA_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29534 bench.py --gpus 4 --steps 20 --warmup 3 --e2e-steps 1 --soak-s 0.1 > gpurun_out/dist4g.json 2>&1

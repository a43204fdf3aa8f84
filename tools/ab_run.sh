cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.txt 2>&1
for r in 1 2; do for v in prev cur; do echo -n "$v "; SAFARA_LIB=$PWD/ablibs/$v.so timeout 300 python bench.py --slab-sim 8 --steps 400 --warmup 10; done; done
for p in 2 4 8; do for g in 0 20; do timeout 300 python bench.py --slab-sim $p --steps 400 --warmup 10 --graph $g; done; done
for p in 2 4 8; do for g in 0 20; do timeout 300 python bench.py --slab-sim $p --config SP-B --steps 400 --warmup 10 --graph $g; done; done
AB_ARGS="" bash tools/ab.sh 400 ablibs/prev.so ablibs/cur.so ablibs/prev.so ablibs/cur.so
SAFARA_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 40 --warmup 3 --e2e-steps 2 --soak-s 0.2 --graph 20 > gpurun_out/dist2g.json 2>&1

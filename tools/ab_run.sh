cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.txt 2>&1
for r in 1 2 3; do AB_ARGS="" bash tools/ab.sh 300 ablibs/cur.so ablibs/one2.so ablibs/cur2.so; done
for cfg in "BT-C 2" "BT-C 4" "BT-C 8" "SP-B 4" "SP-B 8"; do set -- $cfg; timeout 300 python bench.py --slab-sim $2 --config $1 --steps 400 --warmup 10 --graph 20; done > gpurun_out/slabsim_final.txt 2>&1

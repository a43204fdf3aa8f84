cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_peer.py tests/test_gpu_parity.py -q -x > gpurun_out/pytest_peer.txt 2>&1
for cfg in "BT-C 2" "BT-C 4" "BT-C 8" "SP-B 2" "SP-B 4" "SP-B 8"; do set -- $cfg; for b in 0 3; do echo -n "bias $b "; SAFARA_PEER_BIAS=$b timeout 300 python bench.py --slab-sim $2 --config $1 --steps 400 --warmup 10 --graph 20; done; done

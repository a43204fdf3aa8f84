cd $GRAFT_REPO_ROOT
SAFARA_LIB=$PWD/ablibs/idle.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_aux_norm.py -q -x > gpurun_out/pytest_idle.txt 2>&1
for r in 1 2 3; do AB_ARGS="" bash tools/ab.sh 400 ablibs/cur.so ablibs/idle.so; done

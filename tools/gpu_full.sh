cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -q -m gpu -x > gpurun_out/gpu_full.txt 2>&1; echo "exit $?" >> gpurun_out/gpu_full.txt
bash tools/gpu_ncu.sh

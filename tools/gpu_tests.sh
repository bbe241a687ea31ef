cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout ${T:-900} python -m pytest ${TESTS:-tests/test_gpu_parity.py} -q -m gpu ${PYARGS} > gpurun_out/gpu_tests.txt 2>&1
echo "exit $?" >> gpurun_out/gpu_tests.txt

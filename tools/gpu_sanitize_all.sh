# racecheck + synccheck over every GPU parity and fuzz test (slower than gpu_sanitize.sh's selection)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in racecheck synccheck; do
  timeout 1500 $CS --tool $tool --print-limit 20 --error-exitcode 9 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py -q -m gpu -p no:cacheprovider > gpurun_out/sanitize_all_$tool.txt 2>&1
  echo "exit $?" >> gpurun_out/sanitize_all_$tool.txt
done

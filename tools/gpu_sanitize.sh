cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
K="test_scan_and_parse_match_oracle or test_decode_memcpy_h2d_matches_oracle or test_decode_arrays_all_types or test_encode_call or test_encode_replies or test_serve_matches_oracle or test_ring_copy"
for tool in memcheck racecheck synccheck; do
  timeout 1500 $CS --tool $tool --print-limit 20 --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "$K" -p no:cacheprovider > gpurun_out/sanitize_$tool.txt 2>&1
  echo "exit $?" >> gpurun_out/sanitize_$tool.txt
  # the persistent server (one resident CTA polling a mapped doorbell)
  timeout 900 $CS --tool $tool --print-limit 20 --error-exitcode 9 python -m pytest tests/test_gpu_server.py -q -m gpu -x -p no:cacheprovider > gpurun_out/sanitize_server_$tool.txt 2>&1
  echo "exit $?" >> gpurun_out/sanitize_server_$tool.txt
done

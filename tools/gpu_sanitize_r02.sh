# compute-sanitizer memcheck / racecheck / synccheck on the round-2 kernels: the chunked multi-CTA scan
# (tests/test_gpu_chunked_scan.py: regular, irregular, host ring, truncations, capacity stops, fallbacks) and the
# striped memcpys through the three planners (tests/test_gpu_stripe.py), plus the serve parity cases (PDL
# launches, composed reply chunks).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck; do
  timeout 1500 $CS --tool $tool --print-limit 20 --error-exitcode 9 python -m pytest tests/test_gpu_chunked_scan.py \
    tests/test_gpu_stripe.py -q -m gpu -x -p no:cacheprovider \
    -k "resolves_chunked or truncations or frag_limit or zero_length or many_rings or serve_through or seed-1 or big_fragments" \
    > gpurun_out/sanitize_r02_$tool.txt 2>&1
  echo "exit $?" >> gpurun_out/sanitize_r02_$tool.txt
  timeout 900 $CS --tool $tool --print-limit 20 --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -q -m gpu -x \
    -k "test_serve_matches_oracle or test_encode_call or test_encode_replies or batch_requests" -p no:cacheprovider \
    > gpurun_out/sanitize_r02_parity_$tool.txt 2>&1
  echo "exit $?" >> gpurun_out/sanitize_r02_parity_$tool.txt
done

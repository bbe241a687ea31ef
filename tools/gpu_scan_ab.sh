# Chunked-scan check on one B200: parity tests, then the suite's long-window configs with the chunked scan
# (default) and with the one-CTA scan (scan_chunking=1).  Outputs under gpurun_out/.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1
timeout ${T:-900} python -m pytest ${TESTS:-tests/test_gpu_chunked_scan.py} -q -m gpu -x > gpurun_out/scan_tests.txt 2>&1
echo "exit $?" >> gpurun_out/scan_tests.txt
for mode in chunked one_cta; do
  if [ $mode = one_cta ]; then export SUITE_CTX=scan_chunking=1; else unset SUITE_CTX; fi
  SUITE_ONLY=${ONLY:-C3_sweep,C4_typed,NEXT1} timeout 900 python tools/suite.py > gpurun_out/suite_$mode.json 2> gpurun_out/suite_$mode.err
  echo "exit $?" >> gpurun_out/suite_$mode.err
done

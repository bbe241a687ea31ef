# Small-call latency check on one B200: GPU tests (TESTS, default the whole -m gpu suite), then the suite's
# small-call configs and the C3 HtoD probe.  Outputs under gpurun_out/.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1
timeout ${T:-1500} python -m pytest ${TESTS:-tests} -q -m gpu -x > gpurun_out/lat_tests.txt 2>&1
echo "exit $?" >> gpurun_out/lat_tests.txt
SUITE_ONLY=${ONLY:-C1,NEXT3,C3} timeout 900 python tools/suite.py > gpurun_out/lat_suite.json 2> gpurun_out/lat_suite.err
timeout 600 python tools/c3_htod_ab.py ${LOGS:-12,20,26,30} default > gpurun_out/lat_c3ab.json 2> gpurun_out/lat_c3ab.err
echo done > gpurun_out/lat_done.txt

# Re-entry check on one B200: build, the whole -m gpu suite, smoke, the default bench line, the smoke launch list.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1
timeout 1500 python -m pytest tests -q -m gpu -x > gpurun_out/head_tests.txt 2>&1; echo "exit $?" >> gpurun_out/head_tests.txt
python __graft_entry__.py smoke > gpurun_out/head_smoke.txt 2>&1; echo "exit $?" >> gpurun_out/head_smoke.txt
timeout 900 python bench.py > gpurun_out/head_bench.json 2> gpurun_out/head_bench.err; echo "exit $?" >> gpurun_out/head_bench.err
/usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/head_smoke_launches.csv python __graft_entry__.py smoke > gpurun_out/head_ncu_smoke.log 2>&1
SUITE_ONLY=C1,NEXT3,C3 timeout 900 python tools/suite.py > gpurun_out/head_suite.json 2> gpurun_out/head_suite.err
echo done > gpurun_out/head_done.txt

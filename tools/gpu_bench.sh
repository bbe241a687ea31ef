cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python __graft_entry__.py smoke > gpurun_out/smoke.txt 2>&1; echo "exit $?" >> gpurun_out/smoke.txt
timeout ${T:-600} python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "exit $?" >> gpurun_out/bench.err

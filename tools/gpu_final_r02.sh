# Round-2 headline measurements on one B200: smoke, the default bench line (with e2e, sweep and CPU baselines),
# the one-way mixes, the suite (C1-C4, NEXT-1/2/3), and ncu launch lists of bench's timed region and smoke.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1
python __graft_entry__.py smoke > gpurun_out/smoke.txt 2>&1; echo "exit $?" >> gpurun_out/smoke.txt
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 500 > gpurun_out/clocks.csv &
SMI=$!
timeout 900 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err; echo "exit $?" >> gpurun_out/bench_final.err
timeout 600 python bench.py --direction h2d --no-sweep --no-cpu > gpurun_out/bench_h2d.json 2>> gpurun_out/bench_final.err
timeout 600 python bench.py --direction d2h --no-sweep --no-cpu > gpurun_out/bench_d2h.json 2>> gpurun_out/bench_final.err
kill $SMI
timeout 900 python tools/suite.py > gpurun_out/suite_final.json 2> gpurun_out/suite_final.err; echo "exit $?" >> gpurun_out/suite_final.err
NCU=/usr/local/cuda/bin/ncu
$NCU --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/bench_launches.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-sweep --no-cpu > gpurun_out/ncu_bench.log 2>&1
$NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/smoke_launches.csv python __graft_entry__.py smoke > gpurun_out/ncu_smoke.log 2>&1
echo done > gpurun_out/final_done.txt

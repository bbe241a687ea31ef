# Launch list (per-kernel durations, serialised) of a suite selection: SUITE_ONLY=... bash tools/gpu_launches.sh
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
tag=${TAG:-sel}
/usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none ${NCU_EXTRA} --csv \
  --log-file gpurun_out/launches_$tag.csv python tools/suite.py > gpurun_out/suite_$tag.json 2> gpurun_out/suite_$tag.err
echo "exit $?" >> gpurun_out/suite_$tag.err

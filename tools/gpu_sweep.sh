cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout ${T:-900} python tools/sweep.py $SWEEP > gpurun_out/sweep.txt 2> gpurun_out/sweep.err

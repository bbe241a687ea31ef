cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout ${T:-1500} python tools/suite.py > gpurun_out/suite.json 2> gpurun_out/suite.err; echo "exit $?" >> gpurun_out/suite.err

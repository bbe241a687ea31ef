cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
$NCU --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python tools/profile_step.py --steps 3 > gpurun_out/ncu_launch.log 2>&1
$NCU --profile-from-start off --set full --import-source on --clock-control none -k regex:mover -c 1 -o gpurun_out/mover -f python tools/profile_step.py --steps 1 > gpurun_out/ncu_full.log 2>&1
$NCU --profile-from-start off --set full --import-source on --clock-control none -k regex:frame_scan -c 1 -o gpurun_out/scan -f python tools/profile_step.py --steps 1 > gpurun_out/ncu_scan.log 2>&1

# Round-2 ncu evidence on one B200 (outputs in gpurun_out/, summarised by tools/ncu_summary.py --round 2):
#   launches.csv          launch list of a lone C5 serve step with the library defaults (chunked scan)
#   bench_launches.csv    launch list of bench.py itself (pipelined loop, its own configuration)
#   smoke_launches.csv    launch list of __graft_entry__.smoke()
#   mover.ncu-rep         --set full of the mover in bench.py's pipelined configuration
#   walk.ncu-rep / emit.ncu-rep   --set full of the chunked scan's two kernels on the C5 endpoint
#   scan.ncu-rep          --set full of the one-CTA scan (scan_chunking=1) on the C5 endpoint
#   host_step_metrics.csv PCIe / DRAM counters of a zero-copy (host ring) server step
#   front.ncu-rep         --set full of the fused single-CTA front end in smoke() (cold: ncu flushes the caches)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
PS="python tools/profile_step.py"
BENCH_CTX=mover_reserve_ctas=16,mover_tail_tiles=0,scan_chunking=1
$NCU --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv $PS --steps 3 > gpurun_out/ncu_launch.log 2>&1
$NCU --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/bench_launches.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-sweep --no-cpu > gpurun_out/ncu_bench.log 2>&1
$NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/smoke_launches.csv python __graft_entry__.py smoke > gpurun_out/ncu_smoke.log 2>&1
$NCU --profile-from-start off --set full --import-source on --clock-control none -k regex:mover -c 1 -o gpurun_out/mover -f $PS --steps 1 --ctx $BENCH_CTX > gpurun_out/ncu_full.log 2>&1
$NCU --profile-from-start off --set full --import-source on --clock-control none -k regex:chunk_walk -c 1 -o gpurun_out/walk -f $PS --steps 1 > gpurun_out/ncu_walk.log 2>&1
$NCU --profile-from-start off --set full --import-source on --clock-control none -k regex:chunk_emit -c 1 -o gpurun_out/emit -f $PS --steps 1 > gpurun_out/ncu_emit.log 2>&1
$NCU --profile-from-start off --set full --import-source on --clock-control none -k regex:frame_scan -c 1 -o gpurun_out/scan -f $PS --steps 1 --ctx scan_chunking=1 > gpurun_out/ncu_scan.log 2>&1
$NCU --set full --import-source on --clock-control none -k regex:front_small -c 1 -o gpurun_out/front -f python __graft_entry__.py smoke > gpurun_out/ncu_front.log 2>&1
bash tools/gpu_ncu_host.sh
echo done > gpurun_out/ncu_r02_done.txt

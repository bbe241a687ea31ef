# ncu evidence for the zero-copy (host ring) server step: PCIe bytes per mover / scan launch vs wire bytes.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
M=gpu__time_duration.sum,pcie__read_bytes.sum,pcie__write_bytes.sum,dram__bytes_read.sum,dram__bytes_write.sum,pcie__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sectors_aperture_sysmem_op_read.sum,lts__t_sectors_aperture_sysmem_op_write.sum
$NCU --profile-from-start off --metrics $M --clock-control none -k regex:'mover|frame_scan|parse' -c 3 --csv \
  --log-file gpurun_out/host_step_metrics.csv python tools/profile_step.py --steps 1 --host > gpurun_out/ncu_host.log 2>&1
echo "exit $?" >> gpurun_out/ncu_host.log

# Server step traces (tools/server_step_trace.py) for several build variants (prebuilt here: the .so files
# travel).  Outputs under gpurun_out/strace_<n>.txt.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
i=0
while IFS= read -r v; do
  VARIANT="$v" REPS=${REPS:-5} timeout 300 python tools/server_step_trace.py > gpurun_out/strace_$i.txt 2>&1
  echo "variant: $v" >> gpurun_out/strace_$i.txt
  i=$((i+1))
done < ${VARIANTS:-tools/strace_variants.txt}

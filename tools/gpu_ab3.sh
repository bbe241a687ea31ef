# A/B of crk_config mover settings with ONE batch in flight (lone launches): CFGS="name:ctx ..." bash tools/gpu_ab3.sh
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for c in ${CFGS}; do
  n=${c%%:*}; x=${c#*:}
  timeout 300 python bench.py --no-e2e --no-cpu --pipeline 1 --ctx "$x" > gpurun_out/ab3_${n}.json 2> gpurun_out/ab3_${n}.err
done

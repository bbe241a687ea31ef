# A/B of crk_config mover settings on the bench step: CFGS="name:ctx name2:ctx2" bash tools/gpu_ab2.sh
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for i in $(seq ${REPS:-1}); do
  for c in ${CFGS}; do
    n=${c%%:*}; x=${c#*:}
    timeout 300 python bench.py --no-e2e --no-cpu --ctx "$x" > gpurun_out/ab2_${n}_$i.json 2> gpurun_out/ab2_${n}_$i.err
  done
done

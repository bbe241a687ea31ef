# A/B of prebuilt experiment libraries on the bench step: VARIANTS="default a b" REPS=2 bash tools/gpu_ab.sh
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for i in $(seq ${REPS:-2}); do
  for v in ${VARIANTS}; do
    lib=paper_conf_sc_eilingkkflm23_b200/lib/libcrk_$v.so
    [ "$v" = default ] && lib=paper_conf_sc_eilingkkflm23_b200/lib/libcrk.so
    CRK_LIB=$lib timeout 300 python bench.py --no-e2e --no-cpu ${BENCH_ARGS} > gpurun_out/ab_${v}_$i.json 2> gpurun_out/ab_${v}_$i.err
  done
done

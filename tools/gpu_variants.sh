# Runs a suite selection against each prebuilt experiment library lib/libcrk_<v>.so (VARIANTS="a b c").
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for v in ${VARIANTS}; do
  lib=paper_conf_sc_eilingkkflm23_b200/lib/libcrk_$v.so
  [ "$v" = default ] && lib=paper_conf_sc_eilingkkflm23_b200/lib/libcrk.so
  CRK_LIB=$lib timeout ${T:-600} python tools/suite.py > gpurun_out/var_$v.json 2> gpurun_out/var_$v.err
  echo "exit $?" >> gpurun_out/var_$v.err
done

cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for v in p2pp0 p2pp; do python -m paper_conf_iiswc_lica22_b200.build --variant $v > /dev/null; done
VARIANTS="p2pp0 p2pp" W="C2" STEPS=300 bash tools/ab_variants.sh > gpurun_out/x_ab.txt 2>&1
for v in default p2pp0 p2pp; do
  if [ $v = default ]; then unset MG_LIB_VARIANT; else export MG_LIB_VARIANT=$v; fi
  K=coarse W=C2 TAG=x_$v bash tools/gpu_stalls.sh > /dev/null 2>&1
done

# round 2: ket-first digestion with and without K_ac/K_bc run aggregation (kfold: MAKO_KF_AGG=0), band order in both
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
for v in kfold main; do
  L=$v; [ $v = main ] && L=
  MAKO_LIB=$L timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2p_$v.log 2>&1; tail -c 100 gpurun_out/r2p_$v.log
done
MAKO_LIB=kfold timeout 900 python -m pytest tests/test_gpu_jk.py tests/test_gpu_eri_prod.py -q -x > gpurun_out/r2p_tests_kfold.log 2>&1; tail -n 2 gpurun_out/r2p_tests_kfold.log

# round 2: lane-per-ket kernels at 3 / 4 resident CTAs per SM for the 2-CTA classes (pp|ps) (ds|ps) (fs|ps)
# (capa: all three at 3; capb: (ds|ps) (fs|ps) at 4, (pp|ps) at 3) vs main (refactored kernel, no caps)
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
for v in main capa capb; do
  L=$v; [ $v = main ] && L=
  MAKO_LIB=$L timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2x_$v.log 2>&1; tail -c 60 gpurun_out/r2x_$v.log
done
for v in capa capb; do
MAKO_LIB=$v timeout 900 python -m pytest tests/test_gpu_jk.py tests/test_gpu_eri_prod.py -q -x > gpurun_out/r2x_tests_$v.log 2>&1; tail -n 1 gpurun_out/r2x_tests_$v.log
done

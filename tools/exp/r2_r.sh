# round 2: slot-batched kernel with a super-batched R phase (one primitive quartet per lane across several GEMM
# batches): (dp|pp) only (main); also (pp|pp) (fs|pp) (fs|dp) (dp|dp) (fp|pp) (slab2); the ket-first classes
# (dp|ps) (dp|ds) (fs|ds) (fp|ps) (fd|ps) (ds|pp) moved to it (slab3); vs fec4888 (pre)
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
for v in main slab2 slab3; do
  L=$v; [ $v = main ] && L=
  MAKO_LIB=$L timeout 900 python -m pytest tests/test_gpu_jk.py tests/test_gpu_eri_prod.py -q -x > gpurun_out/r2r_tests_$v.log 2>&1; tail -n 1 gpurun_out/r2r_tests_$v.log
done
for v in main slab2 slab3 pre; do
  L=$v; [ $v = main ] && L=
  MAKO_LIB=$L timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2r_$v.log 2>&1; tail -c 100 gpurun_out/r2r_$v.log
done

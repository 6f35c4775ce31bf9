# round 2: band/shell pair order, K_ac/K_bc run aggregation in the lane-per-ket and ket-first kernels (values
# first, then the segmented scan; ket shells loaded at task start): parity suite; per-class bench of main and q0
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/r2o_tests.log 2>&1; tail -n 3 gpurun_out/r2o_tests.log
for v in main q0; do
  L=$v; [ $v = main ] && L=
  MAKO_LIB=$L timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2o_$v.log 2>&1; tail -c 100 gpurun_out/r2o_$v.log
done

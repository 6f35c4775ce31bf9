# round 2: band/shell pair order with K_ac/K_bc aggregation in the lane-per-ket and ket-first kernels only
# (DMMA-family run aggregation compiled out): parity suite; bench per class for main, q0 (plain Q order),
# pre (fec4888 kernels); serial per-class times (MAKO_SERIAL=1) for main and q0
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/r2n_tests.log 2>&1; tail -n 3 gpurun_out/r2n_tests.log
for v in main q0 pre; do
  L=$v; [ $v = main ] && L=
  MAKO_LIB=$L timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2n_$v.log 2>&1; tail -c 100 gpurun_out/r2n_$v.log
done
for v in main q0; do
  L=$v; [ $v = main ] && L=
  MAKO_SERIAL=1 MAKO_LIB=$L timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2n_ser_$v.log 2>&1; tail -c 100 gpurun_out/r2n_ser_$v.log
done

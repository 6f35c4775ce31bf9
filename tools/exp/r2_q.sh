# round 2: lane-per-ket classes in band order (ket permutation; the other classes keep the Q order), K_ac/K_bc
# run aggregation in the lane-per-ket kernel: parity suite; per-class bench of main, q0 (MAKO_TPQ_BAND=0), pre
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/r2q_tests.log 2>&1; tail -n 3 gpurun_out/r2q_tests.log
for v in main q0 pre; do
  L=$v; [ $v = main ] && L=
  MAKO_LIB=$L timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2q_$v.log 2>&1; tail -c 100 gpurun_out/r2q_$v.log
done

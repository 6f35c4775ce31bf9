# experiment driver (gpurun): GPU parity tests, then per-class bench of the default build and of each variant
cd ${GRAFT_REPO_ROOT:-.}
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
tail -3 gpurun_out/gpu_tests.log
timeout 400 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 1 > gpurun_out/bench_val.log 2>&1
for v in ${VARIANTS}; do
  MAKO_LIB=$v timeout 400 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 1 > gpurun_out/bench_$v.log 2>&1
done

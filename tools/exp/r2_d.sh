# round 2: transposed + batched-R variant (rbswap) per class
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
MAKO_LIB=rbswap timeout 600 python -m pytest tests/test_gpu_eri_prod.py -q -s -x > gpurun_out/r2d_tests_rbswap.log 2>&1; tail -2 gpurun_out/r2d_tests_rbswap.log
MAKO_LIB=rbswap timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2d_rbswap.log 2>&1; tail -c 200 gpurun_out/r2d_rbswap.log
./tools/atomics_bench > gpurun_out/r2d_atomics.log 2>&1; cat gpurun_out/r2d_atomics.log

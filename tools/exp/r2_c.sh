# round 2: batched lane-per-quartet R (quartet_block_rb) alone and with the transposed classes
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
MAKO_LIB=rb timeout 600 python -m pytest tests/test_gpu_eri_prod.py tests/test_gpu_eri.py -q -s -x > gpurun_out/r2c_tests_rb.log 2>&1; tail -2 gpurun_out/r2c_tests_rb.log
MAKO_LIB=rb timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2c_rb.log 2>&1; tail -c 200 gpurun_out/r2c_rb.log

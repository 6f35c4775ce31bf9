# round 2: strip digestion (lane-per-ket family) and transposed warp-per-quartet classes, A/B per class
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_eri_prod.py tests/test_gpu_jk.py tests/test_gpu_incremental.py -q -s -x > gpurun_out/r2b_tests_main.log 2>&1; tail -2 gpurun_out/r2b_tests_main.log
MAKO_LIB=swapall timeout 600 python -m pytest tests/test_gpu_eri_prod.py -q -s -x > gpurun_out/r2b_tests_swap.log 2>&1; tail -2 gpurun_out/r2b_tests_swap.log
MAKO_NO_STRIP=1 timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2b_nostrip.log 2>&1; tail -c 200 gpurun_out/r2b_nostrip.log
timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2b_strip.log 2>&1; tail -c 200 gpurun_out/r2b_strip.log
MAKO_LIB=swapall timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2b_swap.log 2>&1; tail -c 200 gpurun_out/r2b_swap.log
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:tpq_strip_kernel<.int.1, .int.1" -c 1 -o gpurun_out/r2b_strip11 python tools/profile_build.py > gpurun_out/r2b_strip11.log 2>&1
ls gpurun_out | grep r2b

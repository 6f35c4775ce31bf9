# round 2: fragment-order E~ copies (new main) vs the staged/unstaged lane-per-ket digestion (pre-fragment libs)
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_eri_prod.py tests/test_gpu_eri.py tests/test_gpu_jk.py -q -x > gpurun_out/r2i_tests.log 2>&1; tail -n 1 gpurun_out/r2i_tests.log
timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2i_main.log 2>&1; tail -c 100 gpurun_out/r2i_main.log
MAKO_LIB=nostage timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2i_nostage.log 2>&1; tail -c 100 gpurun_out/r2i_nostage.log

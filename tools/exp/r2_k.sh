# round 2: fragment-order GEMM2 B operands on/off (nob), main
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2k_main.log 2>&1; tail -c 100 gpurun_out/r2k_main.log
MAKO_LIB=nob timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2k_nob.log 2>&1; tail -c 100 gpurun_out/r2k_nob.log
if [ -f paper_conf_sc_han0jlacz0025_b200/libmako_rbg.so ]; then
MAKO_LIB=rbg timeout 600 python -m pytest tests/test_gpu_eri_prod.py -q -x > gpurun_out/r2k_tests_rbg.log 2>&1; tail -n 1 gpurun_out/r2k_tests_rbg.log
MAKO_LIB=rbg timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2k_rbg.log 2>&1; tail -c 100 gpurun_out/r2k_rbg.log
fi

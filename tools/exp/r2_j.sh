# round 2: validate the final kernel set (fragment-order operands, GEMM2 order fix, staging off)
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r2j_tests.log 2>&1; tail -n 1 gpurun_out/r2j_tests.log
timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2j_main.log 2>&1; tail -c 100 gpurun_out/r2j_main.log
TOOLS=initcheck bash tools/exp/sanitize.sh

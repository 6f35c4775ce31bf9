# register-budget variants: rq (TF32 tier accumulators 144/96 floats), r72 (FP64 L>=8 budget 72 doubles)
cd ${GRAFT_REPO_ROOT:-.}
MAKO_LIB=rq timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 1e30 > gpurun_out/bench_var_rq.log 2>&1
MAKO_LIB=r72 timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/bench_var_r72.log 2>&1
MAKO_LIB=rq timeout 900 python -m pytest tests/test_gpu_quant.py -q -x > gpurun_out/var_rq_tests.log 2>&1; tail -2 gpurun_out/var_rq_tests.log

# session-3 check: GPU parity tests, smoke, default bench with per-class times, launch list
cd ${GRAFT_REPO_ROOT:-.}
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
tail -3 gpurun_out/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 600 python bench.py --class-times > gpurun_out/bench_val.log 2>&1
tail -c 600 gpurun_out/bench_val.log

# row f3 (g functions): GPU parity (g tests first), all GPU tests, smoke, per-class bench
cd ${GRAFT_REPO_ROOT:-.}
timeout 900 python -m pytest tests/test_gpu_g.py -x -q -s > gpurun_out/g_tests.log 2>&1
tail -12 gpurun_out/g_tests.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests_all.log 2>&1
tail -3 gpurun_out/gpu_tests_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 600 python bench.py --class-times --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/bench_g1.log 2>&1
python -c "import json; d=json.loads([l for l in open('gpurun_out/bench_g1.log') if l.startswith('{')][-1]); print(d['s_per_iter'], d['value'], d['mixed_precision']['s_per_iter'])"

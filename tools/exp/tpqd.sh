# lane-per-ket D prefetch: tests, bench with class times
cd ${GRAFT_REPO_ROOT:-.}
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_tests_tpqd.log 2>&1
tail -3 gpurun_out/gpu_tests_tpqd.log
timeout 600 python bench.py --class-times --no-cpu-baseline --steps 3 --warmup 3 --mixed 1e-6 > gpurun_out/bench_tpqd.log 2>&1
python -c "import json; d=json.loads([l for l in open('gpurun_out/bench_tpqd.log') if l.startswith('{')][-1]); print(d['s_per_iter'], d['value'], d['mixed_precision']['s_per_iter'])"

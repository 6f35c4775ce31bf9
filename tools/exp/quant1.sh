# reduced-precision tier: parity tests, then bench with class times and the mixed line
cd ${GRAFT_REPO_ROOT:-.}
timeout 900 python -m pytest tests/test_gpu_quant.py -x -q -s > gpurun_out/quant_tests.log 2>&1
tail -15 gpurun_out/quant_tests.log
timeout 300 python -m pytest tests/test_gpu_eri.py tests/test_gpu_jk.py -x -q > gpurun_out/gpu_tests2.log 2>&1
tail -2 gpurun_out/gpu_tests2.log
for t in 1e-6 1e-4 1e30; do
timeout 400 python bench.py --no-cpu-baseline --steps 2 --warmup 1 --mixed $t > gpurun_out/bench_mixed_$t.log 2>&1
python -c "import json,sys; d=json.loads([l for l in open('gpurun_out/bench_mixed_$t.log') if l.startswith('{')][-1]); print(d['s_per_iter'], d['mixed_precision'])"
done

# row f3 (g functions) parity after the long-double oracle; all GPU tests; g workload bench; FP64 ncu captures
cd ${GRAFT_REPO_ROOT:-.}
timeout 900 python -m pytest tests/test_gpu_g.py -x -q -s > gpurun_out/g_tests.log 2>&1
tail -12 gpurun_out/g_tests.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests_all.log 2>&1
tail -3 gpurun_out/gpu_tests_all.log
timeout 600 python bench.py --config benzene-ccpvqz --class-times --no-cpu-baseline --steps 3 --warmup 3 --mixed 1e-6 > gpurun_out/bench_bzqz.log 2>&1
python -c "import json; d=json.loads([l for l in open('gpurun_out/bench_bzqz.log') if l.startswith('{')][-1]); print(d['s_per_iter'], d['value'], d['mixed_precision']['s_per_iter'])"
for k in 'jk_kernel_free<.int.8, .int.4' 'jk_kernel_capped<.int.8, .int.4' 'jk_kernel_free<.int.9, .int.7' 'jk_kernel_free<.int.7, .int.2' 'slab_jk_kernel<.int.4, .int.2'; do
  n=$(echo "$k" | tr -dc 'a-z0-9')
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:${k}" -c 1 -o gpurun_out/prof64_$n python tools/profile_build.py --nshards 40 --shard 3 > gpurun_out/prof64_$n.log 2>&1
done
ls gpurun_out

# L-dependent R ILP: tests, bench with class times; ncu of the biggest ket-first / lane-per-ket classes
cd ${GRAFT_REPO_ROOT:-.}
timeout 1500 python -m pytest tests/test_gpu_eri.py tests/test_gpu_jk.py tests/test_gpu_g.py -q -x > gpurun_out/gpu_tests_ilp2.log 2>&1
tail -3 gpurun_out/gpu_tests_ilp2.log
timeout 600 python bench.py --class-times --no-cpu-baseline --steps 3 --warmup 3 --mixed 1e-6 > gpurun_out/bench_ilp2.log 2>&1
python -c "import json; d=json.loads([l for l in open('gpurun_out/bench_ilp2.log') if l.startswith('{')][-1]); print(d['s_per_iter'], d['value'], d['mixed_precision']['s_per_iter'])"
for k in 'kf_kernel_capped<.int.4, .int.1' 'tpq_jk_kernel<.int.1, .int.1' 'tpq_jk_kernel<.int.3, .int.1'; do
  n=$(echo "$k" | tr -dc 'a-z0-9')
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:${k}" -c 1 -o gpurun_out/prof_$n python tools/profile_build.py --nshards 40 --shard 3 > gpurun_out/prof_$n.log 2>&1
done

# round 2: new defaults (transposed + batched-R classes, oriented digestion atomics, staged lane-per-ket atomics)
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -s > gpurun_out/r2f_gpu_tests.log 2>&1; tail -n 2 gpurun_out/r2f_gpu_tests.log
timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2f_main.log 2>&1; tail -c 100 gpurun_out/r2f_main.log
for k in 'jk_kernel_free<.int.7, .int.4' 'jk_kernel_free<.int.3, .int.7' 'jk_kernel_free<.int.6, .int.2' 'tpq_jk_kernel<.int.1, .int.1' 'kf_kernel_capped<.int.4, .int.1'; do
  n=$(echo "$k" | tr -dc 'a-z0-9')
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:${k}" -c 1 -o gpurun_out/r2f_$n python tools/profile_build.py > gpurun_out/r2f_$n.log 2>&1
done
ls gpurun_out | grep r2f

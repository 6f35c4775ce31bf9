# round 2, first GPU pass: all GPU tests (incl. the new production-kernel ERI parity), bench per class,
# ncu full captures of the lane-per-ket / ket-first kernels (atomic ceiling)
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -s > gpurun_out/r2a_gpu_tests.log 2>&1; tail -3 gpurun_out/r2a_gpu_tests.log
timeout 900 python bench.py --class-times --no-cpu-baseline --steps 3 --warmup 3 --mixed 0 > gpurun_out/r2a_bench_cls.log 2>&1; tail -c 300 gpurun_out/r2a_bench_cls.log
for k in 'tpq_jk_kernel<.int.1, .int.1' 'tpq_jk_kernel<.int.3, .int.1' 'kf_kernel_capped<.int.4, .int.1' 'jk_kernel_free<.int.7, .int.2'; do
  n=$(echo "$k" | tr -dc 'a-z0-9')
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:${k}" -c 1 -o gpurun_out/r2a_$n python tools/profile_build.py > gpurun_out/r2a_$n.log 2>&1
done
ls gpurun_out

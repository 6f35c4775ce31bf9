# experiment driver (gpurun): ncu --set full captures of the top kernels on a 1/40 shard
cd ${GRAFT_REPO_ROOT:-.}
for k in ${KERNELS:-'jk_kernel_free<.int.7, .int.2>' 'kf_kernel_capped<.int.4, .int.1>' 'tpq_jk_kernel<.int.1, .int.1>' 'jk_kernel_free<.int.4, .int.4>' 'slab_jk_kernel<.int.4, .int.2>' 'jk_kernel_free<.int.9, .int.9>'}; do
  n=$(echo "$k" | tr -dc 'a-z0-9')
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:${k}" -c 1 -o gpurun_out/prof_$n python tools/profile_build.py --nshards 40 --shard 3 > gpurun_out/prof_$n.log 2>&1
done
for v in ${VARIANTS}; do
  MAKO_LIB=$v timeout 400 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 1 > gpurun_out/bench_$v.log 2>&1
done

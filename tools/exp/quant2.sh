# per-class times of the fully-reduced build, ncu captures of TF32-tier vs FP64 kernels (1/40 shard)
cd ${GRAFT_REPO_ROOT:-.}
timeout 400 python bench.py --no-cpu-baseline --steps 1 --warmup 1 --mixed 1e30 --class-times > gpurun_out/bench_q_cls.log 2>&1
for k in 'jk_kernel_q<.int.9, .int.9' 'jk_kernel_q<.int.8, .int.4' 'jk_kernel_free<.int.8, .int.4' 'jk_kernel_q<.int.7, .int.2'; do
  n=$(echo "$k" | tr -dc 'a-z0-9')
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:${k}" -c 1 -o gpurun_out/prof_$n python tools/profile_build.py --nshards 40 --shard 3 --thresh-fp64 1e30 > gpurun_out/prof_$n.log 2>&1
done
ls gpurun_out

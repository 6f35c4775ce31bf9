# round-end evidence: GPU tests, smoke, default bench line (metric + roofline + e2e + cpu_baseline + mixed),
# per-class table (FP64 and fully-reduced TF32 tier), reference arm, g workload, ncu launch list and
# --set full captures (dominant FP64 kernel on a full-build launch; high-l FP64 and TF32-tier kernels)
cd ${GRAFT_REPO_ROOT:-.}
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/final_gpu_tests.log 2>&1; tail -2 gpurun_out/final_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.log 2>&1; tail -1 gpurun_out/final_smoke.log
timeout 900 python bench.py > gpurun_out/final_bench.log 2>&1; tail -c 400 gpurun_out/final_bench.log
timeout 900 python bench.py --class-times --no-cpu-baseline --steps 3 --warmup 3 --mixed 1e30 > gpurun_out/final_bench_cls.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/final_ref.log 2>&1; tail -c 300 gpurun_out/final_ref.log
timeout 600 python bench.py --config benzene-ccpvqz --class-times --no-cpu-baseline --steps 5 --warmup 3 > gpurun_out/final_bench_g.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final_launches.csv python tools/profile_build.py > gpurun_out/final_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:slab_jk_kernel<.int.4, .int.2" -c 1 -o gpurun_out/final_dom python tools/profile_build.py > gpurun_out/final_dom.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:jk_kernel_free<.int.9, .int.8" -c 1 -o gpurun_out/final_ff_fd python tools/profile_build.py > gpurun_out/final_ff_fd.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:jk_kernel_q<.int.9, .int.8" -c 1 -o gpurun_out/final_q_ff_fd python tools/profile_build.py --thresh-fp64 1e30 > gpurun_out/final_q_ff_fd.log 2>&1
ls gpurun_out | grep final

# round 2 final kernels (lane-per-ket caps): GPU suite + smoke, default bench line,
# per-class table, ncu launch list
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r2f3_gpu_tests.log 2>&1; tail -n 1 gpurun_out/r2f3_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2f3_smoke.log 2>&1; tail -n 1 gpurun_out/r2f3_smoke.log
timeout 1200 python bench.py > gpurun_out/r2f3_bench.log 2>&1; tail -c 200 gpurun_out/r2f3_bench.log
timeout 900 python bench.py --class-times --no-cpu-baseline --steps 3 --warmup 3 --mixed 0 > gpurun_out/r2f3_bench_cls.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2f3_launches.csv python tools/profile_build.py > gpurun_out/r2f3_launches.log 2>&1

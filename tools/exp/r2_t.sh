# round 2 (session 3) closing pass on the final picks: GPU suite + smoke, default bench line, per-class table,
# ncu launch list, --set full of the dominant kernel, of a ket-first (dp|ds) and a warp-per-quartet (fp|dp)
# kernel, and the row-f4 Ozaki prototype
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r2t_gpu_tests.log 2>&1; tail -n 1 gpurun_out/r2t_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2t_smoke.log 2>&1; tail -n 1 gpurun_out/r2t_smoke.log
timeout 1200 python bench.py > gpurun_out/r2t_bench.log 2>&1; tail -c 200 gpurun_out/r2t_bench.log
timeout 900 python bench.py --class-times --no-cpu-baseline --steps 3 --warmup 3 --mixed 0 > gpurun_out/r2t_bench_cls.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2t_launches.csv python tools/profile_build.py > gpurun_out/r2t_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:slab_jk_kernel<.int.4, .int.2" -c 1 -o gpurun_out/r2t_dom python tools/profile_build.py > gpurun_out/r2t_dom.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:kf_kernel_capped<.int.4, .int.3|kf_kernel_free<.int.4, .int.3" -c 1 -o gpurun_out/r2t_kf43 python tools/profile_build.py > gpurun_out/r2t_kf43.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:jk_kernel_free<.int.7, .int.4" -c 1 -o gpurun_out/r2t_jk74 python tools/profile_build.py > gpurun_out/r2t_jk74.log 2>&1
for c in ff-ff fd-fd dd-dd; do timeout 300 python tools/ozaki_f64.py --class $c >> gpurun_out/ozaki_r02.jsonl 2>> gpurun_out/ozaki_r02.err; done; tail -n 3 gpurun_out/ozaki_r02.jsonl
ls gpurun_out | grep r2t

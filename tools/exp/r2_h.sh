# round 2 evidence: GPU tests + smoke, default bench line (cpu_baseline, roofline, e2e, clocks, mixed), per-class
# tables, reference arm, C3 + g lines, SCF lines (C2 + row f2), 8-shard balance (C4), ncu launch list and
# --set full of the dominant kernel, Ozaki prototype, sanitizers, C5 one-GPU build with sampled-block parity
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r2h_gpu_tests.log 2>&1; tail -n 1 gpurun_out/r2h_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2h_smoke.log 2>&1; tail -n 1 gpurun_out/r2h_smoke.log
timeout 1200 python bench.py > gpurun_out/r2h_bench.log 2>&1; tail -c 300 gpurun_out/r2h_bench.log
timeout 900 python bench.py --class-times --no-cpu-baseline --steps 3 --warmup 3 --mixed 1e30 > gpurun_out/r2h_bench_cls.log 2>&1
timeout 900 python bench.py --impl reference --steps 5 --warmup 1 > gpurun_out/r2h_ref.log 2>&1; tail -c 300 gpurun_out/r2h_ref.log
timeout 900 python bench.py --config gly10-ccpvtz --steps 5 --warmup 3 > gpurun_out/r2h_bench_c3.log 2>&1; tail -c 200 gpurun_out/r2h_bench_c3.log
timeout 600 python bench.py --config benzene-ccpvqz --class-times --no-cpu-baseline --steps 5 --warmup 3 > gpurun_out/r2h_bench_g.log 2>&1
MAKO_SCF_TIMING=1 timeout 1800 python -m pytest tests/test_gpu_incremental.py -k scf_timing_line -q -s > gpurun_out/r2h_scf.log 2>&1; tail -n 2 gpurun_out/r2h_scf.log
timeout 900 python tools/shard_balance.py --config valinomycin-def2tzvp --nshards 8 --full > gpurun_out/r2h_shards_c4.jsonl 2>&1; tail -n 1 gpurun_out/r2h_shards_c4.jsonl
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2h_launches.csv python tools/profile_build.py > gpurun_out/r2h_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:slab_jk_kernel<.int.4, .int.2" -c 1 -o gpurun_out/r2h_dom python tools/profile_build.py > gpurun_out/r2h_dom.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:jk_kernel_free<.int.9, .int.8" -c 1 -o gpurun_out/r2h_ffdf python tools/profile_build.py > gpurun_out/r2h_ffdf.log 2>&1
for c in ff-ff fd-fd dd-dd; do timeout 300 python tools/ozaki_f64.py --class $c >> gpurun_out/ozaki_r02b.jsonl 2>> gpurun_out/ozaki_r02b.err; done; cat gpurun_out/ozaki_r02b.jsonl
bash tools/exp/sanitize.sh
MAKO_C5=1 timeout 3000 python -m pytest tests/test_gpu_c5.py -q -s > gpurun_out/r2h_c5.log 2>&1; tail -n 3 gpurun_out/r2h_c5.log
ls gpurun_out | grep r2h

# round 2 final evidence: GPU tests + smoke, default bench line (cpu_baseline, roofline, e2e, clocks, mixed),
# per-class table, reference arm, C3 + g lines, 8-shard balance (C4), ncu launch list and --set full of the
# dominant kernel and of the lane-per-ket (ps|ps) kernel, then the C5 one-GPU build with sampled-block parity
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/fin_gpu_tests.log 2>&1; tail -n 1 gpurun_out/fin_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/fin_smoke.log 2>&1; tail -n 1 gpurun_out/fin_smoke.log
timeout 1200 python bench.py > gpurun_out/fin_bench.log 2>&1; tail -c 300 gpurun_out/fin_bench.log
timeout 900 python bench.py --class-times --no-cpu-baseline --steps 3 --warmup 3 --mixed 1e30 > gpurun_out/fin_bench_cls.log 2>&1
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/fin_ref.log 2>&1; tail -c 300 gpurun_out/fin_ref.log
timeout 900 python bench.py --config gly10-ccpvtz --steps 5 --warmup 3 > gpurun_out/fin_bench_c3.log 2>&1; tail -c 200 gpurun_out/fin_bench_c3.log
timeout 600 python bench.py --config benzene-ccpvqz --class-times --no-cpu-baseline --steps 5 --warmup 3 > gpurun_out/fin_bench_g.log 2>&1
timeout 900 python tools/shard_balance.py --config valinomycin-def2tzvp --nshards 8 --full > gpurun_out/fin_shards_c4.jsonl 2>&1; tail -n 1 gpurun_out/fin_shards_c4.jsonl
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/fin_launches.csv python tools/profile_build.py > gpurun_out/fin_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:slab_jk_kernel<.int.4, .int.2" -c 1 -o gpurun_out/fin_dom python tools/profile_build.py > gpurun_out/fin_dom.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:tpq_jk_kernel<.int.1, .int.1" -c 1 -o gpurun_out/fin_tpq11 python tools/profile_build.py > gpurun_out/fin_tpq11.log 2>&1
MAKO_C5=1 timeout 3600 python -m pytest tests/test_gpu_c5.py -q -s > gpurun_out/fin_c5.log 2>&1; tail -n 3 gpurun_out/fin_c5.log
ls gpurun_out | grep fin_

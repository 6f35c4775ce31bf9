# round 2 (session 3) evidence, part 1: GPU tests + smoke, default bench line, per-class table, ncu launch list
# and --set full of the dominant kernel, SCF lines (C2 + row f2), 8-shard balance (C4), sanitizers
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r2l_gpu_tests.log 2>&1; tail -n 1 gpurun_out/r2l_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2l_smoke.log 2>&1; tail -n 1 gpurun_out/r2l_smoke.log
timeout 1200 python bench.py > gpurun_out/r2l_bench.log 2>&1; tail -c 300 gpurun_out/r2l_bench.log
timeout 900 python bench.py --class-times --no-cpu-baseline --steps 3 --warmup 3 --mixed 1e30 > gpurun_out/r2l_bench_cls.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2l_launches.csv python tools/profile_build.py > gpurun_out/r2l_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:slab_jk_kernel<.int.4, .int.2" -c 1 -o gpurun_out/r2l_dom python tools/profile_build.py > gpurun_out/r2l_dom.log 2>&1
MAKO_SCF_TIMING=1 timeout 1800 python -m pytest tests/test_gpu_incremental.py -k scf_timing_line -q -s > gpurun_out/r2l_scf.log 2>&1; tail -n 2 gpurun_out/r2l_scf.log
timeout 900 python tools/shard_balance.py --config valinomycin-def2tzvp --nshards 8 --full > gpurun_out/r2l_shards_c4.jsonl 2>&1; tail -n 1 gpurun_out/r2l_shards_c4.jsonl
bash tools/exp/sanitize.sh
ls gpurun_out | grep -e r2l -e san_ -e scf

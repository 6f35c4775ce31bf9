# cost-balanced shards: GPU tests of the sharded paths, per-rank balance (valinomycin), per-class microbench
cd ${GRAFT_REPO_ROOT:-.}
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests_cb.log 2>&1; tail -2 gpurun_out/gpu_tests_cb.log
timeout 900 python tools/shard_balance.py --config valinomycin-def2tzvp --nshards 8 --full > gpurun_out/shards_val_cb.log 2>&1
tail -1 gpurun_out/shards_val_cb.log
timeout 900 python tools/microbench.py > gpurun_out/microbench.log 2>&1; tail -c 300 gpurun_out/microbench.log
timeout 900 python bench.py --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/bench_cb.log 2>&1; tail -c 200 gpurun_out/bench_cb.log

# modelled-cost shards: sharded-path GPU tests, per-rank balance (valinomycin; ubiquitin 8 shards)
cd ${GRAFT_REPO_ROOT:-.}
timeout 900 python -m pytest tests/test_gpu_jk.py -q > gpurun_out/gpu_tests_cm.log 2>&1; tail -2 gpurun_out/gpu_tests_cm.log
timeout 900 python tools/shard_balance.py --config valinomycin-def2tzvp --nshards 8 --full > gpurun_out/shards_val_cm.log 2>&1
tail -1 gpurun_out/shards_val_cm.log
timeout 2700 python tools/shard_balance.py --config ubiquitin-def2tzvp --nshards 8 > gpurun_out/shards_ubq_cm.log 2>&1
tail -1 gpurun_out/shards_ubq_cm.log

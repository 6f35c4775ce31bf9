# row e evidence on one GPU: per-rank work of 8-way sharded builds (valinomycin-sized, ubiquitin-sized)
cd ${GRAFT_REPO_ROOT:-.}
timeout 900 python tools/shard_balance.py --config valinomycin-def2tzvp --nshards 8 --full > gpurun_out/shards_val.log 2>&1
tail -1 gpurun_out/shards_val.log
timeout 2700 python tools/shard_balance.py --config ubiquitin-def2tzvp --nshards 8 > gpurun_out/shards_ubq.log 2>&1
tail -3 gpurun_out/shards_ubq.log

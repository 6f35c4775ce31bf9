# task-length sweep of the runtime-KT families (warp-per-quartet, slot-batched) on the bench workload
cd ${GRAFT_REPO_ROOT:-.}
for kt in 8 32 4; do
MAKO_KT_EXP=$kt timeout 400 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 3 > gpurun_out/bench_kt$kt.jsonl 2> gpurun_out/bench_kt$kt.err
done

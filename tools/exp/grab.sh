# TASK_GRAB = 2 variant (build.py --variant g2 -D MAKO_TASK_GRAB=2) on the bench workload, per class
cd ${GRAFT_REPO_ROOT:-.}
MAKO_LIB=g2 timeout 400 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 3 > gpurun_out/bench_g2.jsonl 2> gpurun_out/bench_g2.err

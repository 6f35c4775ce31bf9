# round 2: ket-first kernels without any 3-CTA register cap (kfnocap) vs main's list
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
MAKO_LIB=kfnocap timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2kc_kfnocap.log 2>&1; tail -c 60 gpurun_out/r2kc_kfnocap.log

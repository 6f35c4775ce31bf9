# round 2: per-class sweeps of the warp-per-quartet options: batched lane-per-quartet R for every / no class
# (rball, rbnone), GEMM2 B operands from the fragment-order copy for every / no class (fball, fbnone)
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
for v in rball rbnone fball fbnone; do
  MAKO_LIB=$v timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2sw_$v.log 2>&1; tail -c 60 gpurun_out/r2sw_$v.log
done

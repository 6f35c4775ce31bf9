# round 2: warp-per-quartet kernels at 4 CTAs/SM (128-register cap) for every class (jkcap) and for none
# (jknocap), against main's per-class list (fd bras, (fp|dd))
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
for v in jkcap jknocap; do
  MAKO_LIB=$v timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2z_$v.log 2>&1; tail -c 60 gpurun_out/r2z_$v.log
done

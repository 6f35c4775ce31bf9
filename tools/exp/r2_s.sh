# round 2: per-class family re-selection (the picks were measured on older kernels): main; light-ket classes on
# the lane-per-ket kernel where eligible (tpqx); every warp-per-quartet class transposed / none (swapall,
# swapnone); the ket-first classes moved off the ket-first kernel, transposed or not (kfnsa, kfnsn)
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/r2s_tests.log 2>&1; tail -n 1 gpurun_out/r2s_tests.log
for v in main tpqx swapall swapnone kfnsa kfnsn; do
  L=$v; [ $v = main ] && L=
  MAKO_LIB=$L timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2s_$v.log 2>&1; tail -c 60 gpurun_out/r2s_$v.log
done

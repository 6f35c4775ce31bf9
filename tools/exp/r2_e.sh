# round 2: kf/slab classes moved to the warp-per-quartet kernel with batched R (rb2), and transposed (rb2s)
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
for v in rb2 rb2s; do
MAKO_LIB=$v timeout 600 python -m pytest tests/test_gpu_eri_prod.py -q -s -x > gpurun_out/r2e_tests_$v.log 2>&1; tail -1 gpurun_out/r2e_tests_$v.log
MAKO_LIB=$v timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2e_$v.log 2>&1; tail -c 100 gpurun_out/r2e_$v.log
done

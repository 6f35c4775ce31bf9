# round 2: occupancy caps per class: (ps|ps) lane-per-ket at 5 CTAs/SM, the ket-first (dp|ds) (fd|ps) (dd|ps)
# (fs|ds) at 3 CTAs/SM (caps variant) vs main
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
for v in main caps; do
  L=$v; [ $v = main ] && L=
  MAKO_LIB=$L timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2v_$v.log 2>&1; tail -c 60 gpurun_out/r2v_$v.log
done
MAKO_LIB=caps timeout 900 python -m pytest tests/test_gpu_jk.py tests/test_gpu_eri_prod.py -q -x > gpurun_out/r2v_tests_caps.log 2>&1; tail -n 1 gpurun_out/r2v_tests_caps.log
timeout 1200 python tools/microbench.py > gpurun_out/r2v_microbench.jsonl 2> gpurun_out/r2v_microbench.err; tail -c 300 gpurun_out/r2v_microbench.jsonl

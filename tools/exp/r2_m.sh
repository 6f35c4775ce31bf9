# round 2: band/shell pair order + K_ac/K_bc run aggregation (all families) vs the same kernels on the plain
# Q order (q0 variant, MAKO_BAND_W=0): GPU parity suite, per-class bench of both
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/r2m_tests.log 2>&1; tail -n 3 gpurun_out/r2m_tests.log
timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2m_main.log 2>&1; tail -c 300 gpurun_out/r2m_main.log
MAKO_LIB=q0 timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2m_q0.log 2>&1; tail -c 300 gpurun_out/r2m_q0.log

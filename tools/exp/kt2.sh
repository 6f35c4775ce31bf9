# warp-per-quartet KT = 4 default: full GPU suite, default bench line, KT = 2 sweep point
cd ${GRAFT_REPO_ROOT:-.}
timeout 1000 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests_kt4.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests_kt4.log
timeout 400 python bench.py > gpurun_out/bench_final_kt4.jsonl 2> gpurun_out/bench_final_kt4.err
timeout 400 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 3 > gpurun_out/bench_kt4def.jsonl 2> gpurun_out/bench_kt4def.err
MAKO_KT_EXP=2 timeout 400 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 3 > gpurun_out/bench_kt2.jsonl 2> gpurun_out/bench_kt2.err
tail -2 gpurun_out/gpu_tests_kt4.log

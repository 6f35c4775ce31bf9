# round 2: main lib per class; FP64 peaks with clocks; f4 Ozaki prototype; compute-sanitizer over every family
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
timeout 600 python bench.py --class-times --no-cpu-baseline --steps 2 --warmup 2 --mixed 0 > gpurun_out/r2g_main.log 2>&1; tail -c 100 gpurun_out/r2g_main.log
timeout 300 python tools/peaks_fp64_clocks.py > gpurun_out/peaks_fp64_r02.json 2> gpurun_out/peaks_fp64_r02.err; head -c 400 gpurun_out/peaks_fp64_r02.json
for c in ff-ff fd-fd dd-dd; do timeout 300 python tools/ozaki_f64.py --class $c >> gpurun_out/ozaki_r02.jsonl 2>> gpurun_out/ozaki_r02.err; done; cat gpurun_out/ozaki_r02.jsonl
bash tools/exp/sanitize.sh

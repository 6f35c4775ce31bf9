# compute-sanitizer memcheck / racecheck / synccheck / initcheck over tools/sanitize_run.py (every kernel family,
# the density-screened, accumulate, sharded and mixed-precision builds, eri_batch FP64 + TF32)
cd ${GRAFT_REPO_ROOT:-.}
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in ${TOOLS:-memcheck synccheck initcheck}; do
  timeout 1500 $CS --tool $tool --print-limit 20 --error-exitcode 9 python tools/sanitize_run.py > gpurun_out/san_$tool.log 2>&1
  echo "$tool rc=$?"; tail -3 gpurun_out/san_$tool.log
done
# racecheck (shared-memory hazards) on the small workload: still every family's kernels
timeout 2400 $CS --tool racecheck --racecheck-report hazard --print-limit 20 --error-exitcode 9 python tools/sanitize_run.py small > gpurun_out/san_racecheck.log 2>&1
echo "racecheck rc=$?"; tail -3 gpurun_out/san_racecheck.log

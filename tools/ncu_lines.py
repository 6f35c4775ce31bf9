"""Per-source-line summary of an ncu report (needs -lineinfo):
    python tools/ncu_lines.py rep.ncu-rep [top]
Columns: warp-stall samples, instructions executed, L1 shared wavefronts, L1 global tag requests."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows, fname, hdr = [], None, None
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Function Name":
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr and r[0] not in ("",):  # cuda line rows carry the aggregated metrics
        d = dict(zip(hdr[2:], r[2:]))
        def f(k):
            try:
                return float(d.get(k, "0"))
            except ValueError:
                return 0.0
        rows.append((f("Warp Stall Sampling (All Samples)"), f("Instructions Executed"), f("L1 Wavefronts Shared"),
                     f("L1 Tag Requests Global"), fname, r[0], r[1][:90]))
tot = [sum(x[i] for x in rows) for i in range(4)]
print("totals: stall %.3g  inst %.3g  shm_wf %.3g  gl_req %.3g" % tuple(tot))
for x in sorted(rows, reverse=True)[:top]:
    print("%5.1f%% st %5.1f%% in %5.1f%% shw %5.1f%% glr  %s:%s  %s" % (100 * x[0] / max(tot[0], 1), 100 * x[1] / max(tot[1], 1),
          100 * x[2] / max(tot[2], 1), 100 * x[3] / max(tot[3], 1), x[4], x[5], x[6]))

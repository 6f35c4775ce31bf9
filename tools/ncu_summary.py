"""Key counters of ncu --set full captures as JSON (for profiles/):
    python tools/ncu_summary.py rep1.ncu-rep [rep2 ...] > profiles/ncu_rNN_summary.json
Per report: kernel, duration, DRAM bytes read/written, DMMA / HMMA tensor-subpipe instruction rate
(% of peak sustained while active), tensor-pipe and FP64-pipe cycles active (% of elapsed), issue
active, achieved occupancy, registers."""
import csv
import io
import json
import subprocess
import sys

KEYS = {
    "duration": "gpu__time_duration.sum",
    "dram_read": "dram__bytes_read.sum",
    "dram_write": "dram__bytes_write.sum",
    "dmma_inst_pct_active": "sm__inst_executed_pipe_tensor_subpipe_dmma.avg.pct_of_peak_sustained_active",
    "hmma_inst_pct_active": "sm__inst_executed_pipe_tensor_subpipe_hmma.avg.pct_of_peak_sustained_active",
    "tensor_pipe_pct_elapsed": "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
    "fp64_pipe_pct_elapsed": "TPC.TriageCompute.sm__pipe_fp64_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
    "fp64_inst_pct_active": "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
    "issue_active_pct": "sm__issue_active.avg.pct_of_peak_sustained_elapsed",
    "occupancy_pct": "sm__warps_active.avg.pct_of_peak_sustained_active",
    "registers": "launch__registers_per_thread",
}


def summary(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    col = {h: i for i, h in enumerate(hdr)}
    d = {"report": rep.split("/")[-1], "kernel": vals[col["Kernel Name"]] if "Kernel Name" in col else None}
    for k, m in KEYS.items():
        if m in col:
            d[k] = vals[col[m]]
            if units[col[m]]:
                d[k + "_unit"] = units[col[m]]
    return d


if __name__ == "__main__":
    print(json.dumps([summary(r) for r in sys.argv[1:]], indent=1))

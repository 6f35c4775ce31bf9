"""Summarise class_ms of a bench log: python tools/class_report.py gpurun_out/bench_val.log [prev.log]"""
import json
import sys

names = ["ss", "ps", "pp", "ds", "dp", "dd", "fs", "fp", "fd", "ff", "gs", "gp", "gd", "gf", "gg"]


def load(p):
    l = [x for x in open(p) if x.startswith("{")][-1]
    return json.loads(l)


d = load(sys.argv[1])
prev = load(sys.argv[2])["class_ms"] if len(sys.argv) > 2 else {}
print("s/iter", d["s_per_iter"], "TF", d["value"], "dominant", d["roofline"]["kernel"], "frac", d["roofline"]["frac"])
rows = sorted(((v[0], k, v[1] / v[0] / 1e9, v[2], v[3] if len(v) > 3 else 0) for k, v in d["class_ms"].items()),
              reverse=True)
for ms, k, tf, nq, npq in rows[:int(sys.argv[3]) if len(sys.argv) > 3 else 24]:
    pv = prev.get(k, [None])[0]
    extra = f" pq/q={npq/nq:5.1f} ns/pq={ms*1e6/npq:6.3f}" if npq else ""
    print(f"{k:8s} {ms:8.1f} ms {tf:6.2f} TF  ns/q={ms*1e6/nq:6.2f}" + extra + (f"  (was {pv:.1f})" if pv else ""))

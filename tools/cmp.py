"""Compare per-class times of two bench logs: python tools/cmp.py old.log new.log [min_ms]"""
import json
import sys


def load(p):
    return [json.loads(x) for x in open(p) if x.startswith("{")][-1]


a, b = load(sys.argv[1]), load(sys.argv[2])
thr = float(sys.argv[3]) if len(sys.argv) > 3 else 3.0
print("s/iter %.3f -> %.3f   TF %.2f -> %.2f" % (a["s_per_iter"], b["s_per_iter"], a["value"], b["value"]))
ca, cb = a["class_ms"], b["class_ms"]
rows = sorted(ca, key=lambda k: -ca[k][0])
for k in rows:
    x, y = ca[k][0], cb.get(k, [0])[0]
    if abs(x - y) >= thr:
        print("%-8s %8.1f -> %8.1f  (%+6.1f%%)" % (k, x, y, 100 * (y - x) / max(x, 1e-9)))

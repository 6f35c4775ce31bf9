"""Per-class ERI microbenchmark in the paper's E1 setting: shell
quartets per second for every angular-momentum class, no screening, synthetic shells.

    python tools/microbench.py [--centers 32] [--degrees 1,5] > profiles/microbench_r01.jsonl

For contraction degree k, a basis of C random centres U[-2,2]^3 bohr with one shell of each l <= 3 per
centre, k primitives per shell (exponents log-U[0.1,10], seed 0) -- so K_AB = K_CD = k^2 primitive
pairs per shell pair (reading R11 counts primitive pairs; "{k,k}" here = k primitives on every shell).
One J/K build at tau = 0 (every canonical quartet, Schwarz off) through mako_build_jk; per-class
device time from the library's CUDA events (mako_profile_*), per-class quartets and algorithmic FLOPs
from mako_pairs_class_flops.  One JSON line per degree."""
import argparse
import json
import math
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import mako_inputs as mi  # noqa: E402
from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs, build_jk  # noqa: E402

NAMES = ["ss", "ps", "pp", "ds", "dp", "dd", "fs", "fp", "fd", "ff", "gs", "gp", "gd", "gf", "gg"]


def basis(centers, k, seed=0):
    rng = np.random.default_rng(seed)
    xyz = rng.uniform(-2, 2, size=(centers, 3))
    at, ls, nps, ex, cf = [], [], [], [], []
    for a in range(centers):
        for l in range(4):
            at.append(a); ls.append(l); nps.append(k)
            ex += list(np.sort(np.exp(rng.uniform(np.log(0.1), np.log(10.0), k)))[::-1])
            cf += list(rng.uniform(0.2, 1.0, k))
    sh = mi.Shells(np.array(at, np.int32), np.array(ls, np.int32), np.array(nps, np.int32), xyz[np.array(at)],
                   np.array(ex), np.array(cf))
    return sh, np.ones(centers, np.int32), xyz


def run(centers, k, peak):
    sh, Z, xyz = basis(centers, k)
    P = Pairs(Basis(Z, xyz, sh), 0.0)
    D = torch.tensor(mi.synthetic_density(sh.nbf(), max(1, sh.nbf() // 4), seed=0), device="cuda")
    J, K = build_jk(P, D)  # warm-up
    torch.cuda.synchronize()
    P.profile(True)
    build_jk(P, D, J=J, K=K)
    ms, n = P.profile_read()
    P.profile(False)
    fl, q = P.class_flops()
    rows = {}
    for c in range(len(ms)):
        if n[c] == 0 or q[c] == 0:
            continue
        X = (math.isqrt(8 * c + 1) - 1) // 2
        Y = c - X * (X + 1) // 2
        rows[f"({NAMES[X]}|{NAMES[Y]})"] = {"quartets": int(q[c]), "ms": round(float(ms[c]), 4),
                                            "quartets_per_s": float(q[c] / (ms[c] * 1e-3)),
                                            "tflops": float(fl[c] / (ms[c] * 1e-3) / 1e12),
                                            "frac_dmma_peak": float(fl[c] / (ms[c] * 1e-3) / 1e12 / peak)}
    return {"degree": [k, k], "K_AB": k * k, "centers": centers, "nbf": sh.nbf(), "tau": 0.0,
            "total_ms": float(ms.sum()), "classes": rows}


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--centers", type=int, default=32)
    ap.add_argument("--degrees", default="1,5")
    a = ap.parse_args()
    peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles",
                                       "peaks_fp64_r01.json")))["dmma_m16n8k4_tflops"]
    for k in [int(x) for x in a.degrees.split(",")]:
        print(json.dumps(run(a.centers if k == 1 else max(8, a.centers // 2), k, peak)), flush=True)

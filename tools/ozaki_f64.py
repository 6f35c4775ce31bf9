"""Row f4 (exploratory): FP64 GEMM emulated on INT8 tensor cores (Ozaki-style error-free splitting),
measured on the shape of the warp-per-quartet GEMM1 of a high-l class, against FP64.

    python tools/ozaki_f64.py [--class ff-ff] [--kets 2048] [--slices 8] > gpurun_out/ozaki.json

Shape (Eq. 7): one bra pair's E~_ab [n_ab x nH_ab] times the
[p|q] matrices of many kets side by side, [nH_ab x (kets * nH_cd)] -- the batching a task (bra pair,
kets) allows.  Inputs are synthetic with the dynamic range of the real operands: E~ entries spread over
~6 decades, [p|q] = (-1)^|q| R_{p+q} with R from random Hermite-like magnitudes over ~8 decades.

Scheme (Ozaki et al.'s splitting, int8 digits): rows of A and columns of B are scaled by powers of two to
|x| < 1 and cut into s base-128 digit slices D_t (int8, |D_t| <= 127); A B = sum_{t,u} 128^{-(t+u)} D^A_t D^B_u
with every D^A_t D^B_u exact in int32 (k * 127^2 < 2^31).  Keeping t + u <= s + 1 (s(s+1)/2 INT8 GEMMs)
truncates at ~128^{-(s+1)} k max|A_i.| max|B_.j| -- relative to the row/column MAXIMA, so operands whose
entries spread over many decades inside a row (E~ and R do) need more slices than the 53 bits suggest:
a CPU emulation of this script gives 7e-14 |A||B| at s = 8 and 4e-16 at s = 9 (FP64 DGEMM: 1e-15).
The INT8 GEMMs here are torch._int_mm (cuBLASLt; tcgen05 kind::i8 on sm_100a): a feasibility
measurement for the exploratory row, not a product kernel; the J/K path stays FP64 DMMA.
Reports: max relative error vs an exact (float128-accumulated, numpy longdouble) reference on a sample
of columns, the same for the FP64 GEMM, and the times of (a) the INT8 GEMMs alone, (b) the splitting +
recombination, (c) the FP64 GEMM (cuBLAS DGEMM) of the same shape.
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SHAPES = {"ff-ff": (49, 84, 84), "fd-fd": (35, 56, 56), "dd-dd": (25, 35, 35), "fp-pp": (21, 35, 10)}


def pad8(x):
    return (x + 7) // 8 * 8


def split(M, s, dim):
    """M (float64) -> (scale exponents, [s] int8 digit slices) along rows (dim=1) or columns (dim=0)."""
    amax = M.abs().amax(dim=dim, keepdim=True).clamp_min(1e-300)
    e = torch.floor(torch.log2(amax)) + 1.0  # |M 2^-e| < 1
    R = M * torch.exp2(-e)
    out = []
    for _ in range(s):
        R = R * 128.0
        D = torch.clamp(torch.round(R), -127, 127)
        R = R - D
        out.append(D.to(torch.int8))
    return e, out


def ozaki_gemm(A, B, s):
    ea, As = split(A, s, 1)
    eb, Bs = split(B, s, 0)
    C = torch.zeros((A.shape[0], B.shape[1]), dtype=torch.float64, device=A.device)
    for d in range(s + 1, 1, -1):  # small diagonals first
        acc = None
        for t in range(1, d):
            u = d - t
            if t > s or u > s:
                continue
            p = torch._int_mm(As[t - 1], Bs[u - 1])
            acc = p if acc is None else acc + p
        C += acc.to(torch.float64) * (128.0 ** -d)
    return C * torch.exp2(ea) * torch.exp2(eb)


def int_gemms_only(As, Bs, s):
    for d in range(s + 1, 1, -1):
        for t in range(1, d):
            u = d - t
            if t <= s and u <= s:
                torch._int_mm(As[t - 1], Bs[u - 1])


def timed(fn, reps=10):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    fn()
    torch.cuda.synchronize()
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--class", dest="cls", default="ff-ff", choices=sorted(SHAPES))
    ap.add_argument("--kets", type=int, default=2048)
    ap.add_argument("--slices", type=int, default=9)
    ap.add_argument("--seed", type=int, default=0)
    a = ap.parse_args()
    nab, hab, hcd = SHAPES[a.cls]
    m, k, n = max(pad8(nab), 32), (hab + 31) // 32 * 32, pad8(hcd * a.kets)  # cuBLASLt int8: k % 32 (measured)
    g = torch.Generator(device="cuda").manual_seed(a.seed)
    A = torch.zeros((m, k), dtype=torch.float64, device="cuda")
    A[:nab, :hab] = torch.randn((nab, hab), generator=g, device="cuda", dtype=torch.float64) * \
        torch.exp(torch.rand((nab, hab), generator=g, device="cuda", dtype=torch.float64) * -14.0)
    B = torch.zeros((k, n), dtype=torch.float64, device="cuda")
    B[:hab, :hcd * a.kets] = torch.randn((hab, hcd * a.kets), generator=g, device="cuda", dtype=torch.float64) * \
        torch.exp(torch.rand((hab, hcd * a.kets), generator=g, device="cuda", dtype=torch.float64) * -18.0)
    C64 = A @ B
    res = {"class": a.cls, "shape_mkn": [m, k, n], "slices": a.slices, "int8_gemms": a.slices * (a.slices + 1) // 2}
    for s in sorted({a.slices - 2, a.slices, a.slices + 1}):
        Coz = ozaki_gemm(A, B, s)
        # exact reference on a column sample (long double accumulation of the exact products)
        cols = np.random.default_rng(a.seed).choice(n, 64, replace=False)
        Ah = A.cpu().numpy().astype(np.longdouble)
        Bh = B.cpu().numpy()[:, cols].astype(np.longdouble)
        ref = Ah @ Bh
        scale = np.abs(Ah) @ np.abs(Bh)
        ok = scale > 0
        err_oz = np.abs(Coz.cpu().numpy()[:, cols] - ref)[ok] / scale[ok]
        err_64 = np.abs(C64.cpu().numpy()[:, cols] - ref)[ok] / scale[ok]
        res[f"s{s}"] = {"max_err_over_absAabsB": float(err_oz.max()), "fp64_max_err_over_absAabsB": float(err_64.max())}
    flop = 2.0 * m * k * n
    ea, As = split(A, a.slices, 1)
    eb, Bs = split(B, a.slices, 0)
    t_int = timed(lambda: int_gemms_only(As, Bs, a.slices))
    t_oz = timed(lambda: ozaki_gemm(A, B, a.slices))
    t_64 = timed(lambda: A @ B)
    res.update({"ms_int8_gemms": t_int, "ms_ozaki_total": t_oz, "ms_fp64_dgemm": t_64,
                "fp64_equiv_tflops_int8_part": flop / (t_int * 1e-3) / 1e12,
                "fp64_equiv_tflops_total": flop / (t_oz * 1e-3) / 1e12, "dgemm_tflops": flop / (t_64 * 1e-3) / 1e12})
    print(json.dumps(res))


if __name__ == "__main__":
    main()

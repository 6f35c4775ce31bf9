#!/usr/bin/env python
"""bench.py -- BASELINE.json metric "Fock J+K build s/iter & ERI contraction TFLOP/s at 1/2/4/8 B200".

A step = one direct-SCF J/K build (mako_build_jk: all angular-momentum classes (55 for the l <= 3 bases benched) -- Boys, R
recursion, the two DMMA Hermite->AO contractions, FP64 digestion -- plus, for N > 1, broadcast(D)
and all_reduce(J, K)) over the valinomycin-sized def2-TZVP workload (BASELINE.json configs[3],
"J/K build at 1/2/4/8 GPUs"; configs[4] is an 8-GPU-only config and configs[0..2] are parity cases).

  value       ERI-contraction TFLOP/s: algorithmic FP64 FLOPs of PAPER.md Eq. 7 (a7 + a8) over all
              surviving canonical quartets (unpadded spherical dims, DESIGN.md S Measurement)
              / device time per build (max over ranks).  Whole job over N GPUs.
  s_per_iter  the same build time in seconds (the metric's first half).
  e2e         the same metric through the public API with D copied from pinned host memory and
              J, K read back every step (host<->device copies inside the timed region).

Usage:  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl mako|reference]
        torchrun --nproc-per-node N bench.py --gpus N ...
"""
import argparse
import json
import math
import os
import subprocess
import sys
import tempfile
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import mako_inputs as mi  # noqa: E402

METRIC = "Fock J+K build s/iter & ERI contraction TFLOP/s at 1/2/4/8 B200"
UNIT = "TFLOP/s"
DEFAULT_CONFIG = "valinomycin-def2tzvp"
TAU = 1e-12
PRIM_EPS = 1e-18  # primitive-pair rule of include/mako.h (reading R7)


def peaks():
    p = os.path.join(ROOT, "profiles", "peaks_fp64_r02.json")
    d = json.load(open(p))
    return d


# ---------------------------------------------------------------------------------------------
# workload accounting in Python (used by the reference arm; cross-checked against the library)
# ---------------------------------------------------------------------------------------------
def _nH(L):
    return (L + 1) * (L + 2) * (L + 3) // 6


def workload_flops(sh, Q, tau, prim_eps=PRIM_EPS):
    """Algorithmic FLOPs of a7+a8 over the canonical quartets surviving Q_ab Q_cd >= tau, with the
    library's class orientation (bra = higher (la,lb) bucket).  Q: [nshell, nshell] Schwarz table."""
    poff = np.concatenate([[0], np.cumsum(sh.nprim)])
    buckets = {}
    for a in range(sh.nshell):
        for b in range(sh.nshell):
            la, lb = int(sh.l[a]), int(sh.l[b])
            if la < lb or (la == lb and a < b):
                continue
            R2 = float(np.sum((sh.xyz[a] - sh.xyz[b]) ** 2))
            ea = sh.exps[poff[a]:poff[a + 1]][:, None]
            eb = sh.exps[poff[b]:poff[b + 1]][None, :]
            K = int(np.count_nonzero(np.exp(-ea * eb / (ea + eb) * R2) >= prim_eps))
            if K == 0:
                continue
            buckets.setdefault(la * (la + 1) // 2 + lb, []).append((Q[a, b], K))
    qmax = max(q for v in buckets.values() for q, _ in v)
    # library order: primitive-count group, then Q descending (csrc/mako_internal.h kgroup)
    def kgroup(K):
        return K - 1 if K <= 4 else (4 if K <= 6 else 5 if K <= 9 else 6 if K <= 12 else 7 if K <= 16 else
                                     8 if K <= 24 else 9 if K <= 36 else 10)
    for k in list(buckets):
        v = sorted([x for x in buckets[k] if x[0] * qmax >= tau], key=lambda x: (kgroup(x[1]), -x[0]))
        buckets[k] = (np.array([x[0] for x in v]), np.array([x[1] for x in v], np.int64),
                      np.array([kgroup(x[1]) for x in v], np.int64))
    bl = lambda b: [(la, lb) for la in range(5) for lb in range(la + 1)][b]
    total, nq = 0.0, 0
    for X in buckets:
        for Y in buckets:
            if Y > X:
                continue
            QX, KX, GX = buckets[X]
            QY, KY, GY = buckets[Y]
            la, lb = bl(X)
            lc, ld = bl(Y)
            nab, ncd = (2 * la + 1) * (2 * lb + 1), (2 * lc + 1) * (2 * ld + 1)
            hab, hcd = _nH(la + lb), _nH(lc + ld)
            cK = np.concatenate([[0], np.cumsum(KY)])
            for g in range(11):
                s0, s1 = np.searchsorted(GY, g, "left"), np.searchsorted(GY, g, "right")
                if s1 <= s0:
                    continue
                seg = QY[s0:s1]
                # kets of the group with QP * Q >= tau: prefix of the descending segment
                cnt = np.array([np.searchsorted(-(qp * seg), -tau, side="right") for qp in QX], np.int64)
                if X == Y:  # canonical: ket position <= bra position
                    cnt = np.minimum(cnt, np.maximum(0, np.arange(len(QX)) - s0 + 1))
                sK = cK[s0 + cnt] - cK[s0]
                total += float(np.sum(KX * sK) * 2.0 * nab * hab * hcd + np.sum(sK) * 2.0 * nab * hcd * ncd)
                nq += int(cnt.sum())
    return total, nq


# ---------------------------------------------------------------------------------------------
# clocks during the timed region (B200_PROFILING.md clocks line)
# ---------------------------------------------------------------------------------------------
class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.proc = None
        self.file = None

    def start(self):
        try:
            self.file = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), "--query-gpu=" + self.FIELDS,
                                          "--format=csv,noheader,nounits", "-lms", "200"], stdout=self.file,
                                         stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(5)
        except Exception:
            self.proc.kill()
        self.file.flush()
        self.file.seek(0)
        rows = [r.strip().split(", ") for r in self.file.read().strip().splitlines() if r.strip()]
        os.unlink(self.file.name)
        sm = [float(r[1]) for r in rows if len(r) >= 9 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if len(r) >= 9 and r[2].replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            if len(r) < 9:
                continue
            for nm, v in zip(names, r[5:9]):
                if v.strip() == "Active":
                    reasons.add(nm)
        loaded = [s for s in sm if s > 0.5 * max(sm)] if sm else []
        return {"sm_mhz": float(np.median(loaded)) if loaded else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(rows)}


# ---------------------------------------------------------------------------------------------
# CPU baseline: the oracle as it stands, on a bounded sample of the same workload
# ---------------------------------------------------------------------------------------------
def _nquartet_index(sh):
    npair = sh.nshell * (sh.nshell + 1) // 2
    return npair * (npair + 1) // 2  # canonical quartet indices P(P+1)/2 + R, R <= P < npair


def oracle_overhead(sh, D, tau, Q):
    """Per-call cost of the oracle J/K that does not scale with the sample (per-thread nbf^2 accumulators,
    their reduction, the symmetrisation): one call on an empty quartet sample (shard index beyond the
    last canonical quartet).  A full build pays it once."""
    import oracle
    nidx = _nquartet_index(sh)
    t0 = time.perf_counter()
    oracle.jk_qsample(sh, D, tau, nidx, nidx + 1, Q=Q)
    return time.perf_counter() - t0


def oracle_sample_seconds(sh, D, tau, Q, target_s, first_shard=0):
    """Size a uniform quartet sample (canonical quartet index % S == shard, orc_jk_qsample: every class and
    every bra pair sampled alike, so the spread between samples is small) so that its WORK (call time
    minus the per-call overhead) is about target_s; returns (S, overhead_s).  S < 2: the whole build fits."""
    import oracle
    nidx = _nquartet_index(sh)
    ovh = oracle_overhead(sh, D, tau, Q)
    S0 = max(2, min(nidx, 40000))  # pilot samples of a few seconds: the work dominates the overhead
    t0 = time.perf_counter()
    for i in range(2):
        oracle.jk_qsample(sh, D, tau, (first_shard + i * (S0 // 2) + 1) % S0, S0, Q=Q)
    work = max((time.perf_counter() - t0) / 2 - ovh, 1e-4)
    S = int(min(work * S0 / target_s, nidx))
    return S, ovh


def oracle_sampled_build(sh, D, tau, Q, S, shard, ovh):
    """One timed oracle call on the quartet sample shard/S; extrapolated full-build seconds
    (work x S + the per-call overhead once)."""
    import oracle
    t0 = time.perf_counter()
    oracle.jk_qsample(sh, D, tau, shard, S, Q=Q)
    ts = time.perf_counter() - t0
    return ts, max(ts - ovh, 0.0) * S + ovh


def cpu_baseline(sh, D, tau, total_flops, target_s=15.0, Q=None):
    import oracle
    if Q is None:
        Q = oracle.schwarz(sh)
    S, ovh = oracle_sample_seconds(sh, D, tau, Q, target_s)
    if S < 2:  # the whole build fits the budget: time it directly
        t0 = time.perf_counter()
        oracle.jk(sh, D, tau, Q=Q)
        ts = time.perf_counter() - t0
        return {"value": total_flops / ts / 1e12, "unit": UNIT, "cores": oracle.num_threads(), "kind": "oracle",
                "sample": f"the full build, {ts:.1f} s", "s_per_iter": ts, "extrapolated": False}
    shard = S // 2
    ts, s_per_build = oracle_sampled_build(sh, D, tau, Q, S, shard, ovh)
    return {"value": total_flops / s_per_build / 1e12, "unit": UNIT, "cores": oracle.num_threads(), "kind": "oracle",
            "sample": f"canonical shell quartets with quartet_index % {S} == {shard} (1/{S} of the build, every "
                      f"class sampled uniformly): {ts:.1f} s measured, per-call overhead {ovh:.2f} s (empty-sample "
                      f"call) counted once, work x{S}",
            "s_per_iter_extrapolated": s_per_build, "sample_s": ts, "overhead_s": ovh, "extrapolated": True}


# ---------------------------------------------------------------------------------------------
def run_reference(args):
    """--impl reference: the oracle (plain C, OpenMP) timed on the host cores, rank 0 only.  Each step is
    one strided sample of canonical bra pairs (a different shard per step), sized and extrapolated exactly
    as bench.py's cpu_baseline leg (per-call overhead measured on an empty shard and counted once)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    mol, basis = mi.config_molecule(args.config)
    sh = mi.shells_for(mol, basis)
    n = sh.nbf()
    D = mi.synthetic_density(n, mol.nelec // 2, seed=0)
    Q = oracle.schwarz(sh)
    total, nq = workload_flops(sh, Q, args.tau)
    S, ovh = oracle_sample_seconds(sh, D, args.tau, Q, args.ref_step_s)
    S = max(S, 2)
    builds, samples = [], []
    for i in range(args.warmup + args.steps):
        shard = (7 * i + S // 2) % S
        ts, sb = oracle_sampled_build(sh, D, args.tau, Q, S, shard, ovh)
        if i >= args.warmup:
            builds.append(sb)
            samples.append(ts)
    s_per_build = float(np.mean(builds))
    value = total / s_per_build / 1e12
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": s_per_build * 1e3, "higher_is_better": True,
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
            "extrapolated": True, "sample_s_per_step": samples, "overhead_s": ovh,
            "config": {"workload": args.config, "basis": mi.basis_label(basis), "nbf": n, "tau": args.tau,
                       "quartets": nq, "gemm_flops_per_build": total},
            "s_per_iter": s_per_build,
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": oracle.num_threads(), "kind": "oracle",
                             "sample": f"each step: canonical shell quartets with index % {S} == shard (1/{S} of "
                                       f"the build, shards vary per step; {np.mean(samples):.1f} s measured per "
                                       f"step), work x{S} + per-call overhead {ovh:.2f} s once (extrapolated)"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def run_mako(args):
    import torch
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        if rank == 0:
            print(f"warning: --gpus {args.gpus} but WORLD_SIZE={world}; using WORLD_SIZE", file=sys.stderr)
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    from paper_conf_sc_han0jlacz0025_b200 import Basis, Pairs, build_jk
    from paper_conf_sc_han0jlacz0025_b200.mako import FAMILY_KERNELS, class_family, class_reduced
    from paper_conf_sc_han0jlacz0025_b200.dist import combine_jk

    mol, basis = mi.config_molecule(args.config)
    sh = mi.shells_for(mol, basis)
    n = sh.nbf()
    stream = torch.cuda.current_stream()
    t0 = time.perf_counter()
    B = Basis(mol.Z, mol.xyz_bohr, sh)
    P = Pairs(B, args.tau)
    pair_s = time.perf_counter() - t0
    stats = P.stats()
    flops_total = P.flops()["gemm_flops"]
    cls_flops, cls_q = P.class_flops(shard=rank, nshards=world)
    launches_per_build = P.launches(shard=rank, nshards=world)

    Dh = mi.synthetic_density(n, mol.nelec // 2, seed=0)
    D = torch.tensor(Dh, device="cuda")
    J = torch.empty_like(D)
    K = torch.empty_like(D)

    def step():
        if world > 1:
            dist.broadcast(D, src=0)
        build_jk(P, D, J=J, K=K, shard=rank, nshards=world, stream=stream)
        if world > 1:
            combine_jk(J, K)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    P.profile(True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        step()
    e1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ms = e0.elapsed_time(e1) / args.steps
    cls_ms, cls_n = P.profile_read()
    P.profile(False)
    clk = clocks.stop()
    if world > 1:
        t = torch.tensor([ms], device="cuda", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    value = flops_total / (ms * 1e-3) / 1e12

    # stage-aware reduced-precision tier (mako_build_jk_mixed): same workload, quartets
    # with Q_ab Q_cd max|D| < thresh_fp64 in the TF32 tier; error of the two-electron energy vs FP64
    mixed = None
    names_ = ["ss", "ps", "pp", "ds", "dp", "dd", "fs", "fp", "fd", "ff", "gs", "gp", "gd", "gf", "gg"]
    if args.mixed > 0 and world == 1:
        Jm, Km = torch.empty_like(D), torch.empty_like(D)
        build_jk(P, D, J=Jm, K=Km, stream=stream, thresh_fp64=args.mixed)
        torch.cuda.synchronize()
        nm = max(1, min(args.steps, 3))
        e0.record(stream)
        for _ in range(nm):
            build_jk(P, D, J=Jm, K=Km, stream=stream, thresh_fp64=args.mixed)
        e1.record(stream)
        torch.cuda.synchronize()
        ms_m = e0.elapsed_time(e1) / nm
        cls_ms_m = None
        if args.class_times:
            P.profile(True)
            build_jk(P, D, J=Jm, K=Km, stream=stream, thresh_fp64=args.mixed)
            cls_ms_m, _ = P.profile_read()
            P.profile(False)
        e2 = lambda JJ, KK: 0.5 * float(torch.sum(D * (JJ - 0.5 * KK)))
        mixed = {"thresh_fp64": args.mixed, "s_per_iter": ms_m * 1e-3, "value": flops_total / (ms_m * 1e-3) / 1e12,
                 "unit": UNIT, "speedup_vs_fp64": ms / ms_m, "steps": nm,
                 "dE2_vs_fp64_Ha": e2(Jm, Km) - e2(J, K),
                 "max_dJ": float((Jm - J).abs().max()), "max_dK": float((Km - K).abs().max()),
                 "tiers": "FP64 Boys/R + TF32 GEMM1/GEMM2 (FP32 accumulate) + FP64 digestion for quartets with "
                          "Q_ab Q_cd max|D| < thresh_fp64 in the %d classes with a reduced kernel; FP64 otherwise"
                          % int(class_reduced().sum())}
        if cls_ms_m is not None:
            mixed["class_ms"] = {f"({names_[int((math.isqrt(8*i+1)-1)//2)]}|"
                                 f"{names_[i - int((math.isqrt(8*i+1)-1)//2) * (int((math.isqrt(8*i+1)-1)//2) + 1) // 2]})":
                                 round(float(cls_ms_m[i]), 4) for i in range(len(cls_ms_m)) if cls_ms_m[i] > 0}
        del Jm, Km

    # end to end through the public API with host buffers (pinned), copies inside the timed region
    Dpin = torch.from_numpy(Dh).pin_memory()
    Jpin = torch.empty((n, n), dtype=torch.float64).pin_memory()
    Kpin = torch.empty((n, n), dtype=torch.float64).pin_memory()

    def e2e_step():
        D.copy_(Dpin, non_blocking=True)
        step()
        Jpin.copy_(J, non_blocking=True)
        Kpin.copy_(K, non_blocking=True)

    e2e_steps = max(1, min(args.steps, 3))
    e2e_step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    e0.record(stream)
    for _ in range(e2e_steps):
        e2e_step()
    e1.record(stream)
    torch.cuda.synchronize()
    ms_e2e = e0.elapsed_time(e1) / e2e_steps
    if world > 1:
        t = torch.tensor([ms_e2e], device="cuda", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_e2e = float(t.item())

    # roofline of the dominant kernel (largest device time share among the class kernels)
    pk = peaks()
    c = int(np.argmax(cls_ms))
    per_launch_ms = cls_ms[c] / max(cls_n[c], 1)
    achieved = cls_flops[c] / (per_launch_ms * 1e-3) / 1e12
    names = ["ss", "ps", "pp", "ds", "dp", "dd", "fs", "fp", "fd", "ff", "gs", "gp", "gd", "gf", "gg"]
    X = int((math.isqrt(8 * c + 1) - 1) // 2)
    Y = c - X * (X + 1) // 2
    traffic = None
    tp = os.path.join(ROOT, "profiles", "ncu_dominant.json")
    if os.path.exists(tp):
        try:
            tj = json.load(open(tp))
            if tj.get("class") == f"({names[X]}|{names[Y]})" and tj.get("config") == args.config:
                traffic = tj.get("dram_bytes_per_launch")
        except Exception:
            traffic = None
    roof = {"bound": "tensor", "achieved": achieved, "peak": pk["dmma_m16n8k4_tflops"], "unit": "TFLOP/s",
            "frac": achieved / pk["dmma_m16n8k4_tflops"], "traffic": traffic,
            "kernel": f"{FAMILY_KERNELS[int(class_family()[c])]}<{X},{Y}> class ({names[X]}|{names[Y]})",
            "share_of_step": float(cls_ms[c] / max(cls_ms.sum(), 1e-9)),
            "peak_source": "FP64 DMMA mma.sync m16n8k4 loop measured on this pool's B200 with the clock record "
                           "(profiles/peaks_fp64_r02.json: 1965 MHz, no throttle reason; MEASURED_PEAKS.json "
                           "has no FP64 entry)",
            "all_classes_achieved": value / world, "all_classes_frac": value / world / pk["dmma_m16n8k4_tflops"]}

    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": args.config, "basis": mi.basis_label(basis), "atoms": mol.natm, "nbf": n,
                       "shells": sh.nshell, "tau": args.tau, "pairs": stats["pairs"], "prim_pairs": stats["prim_pairs"],
                       "quartets": stats["quartets"], "gemm_flops_per_build": flops_total,
                       "parallelism": f"quartet-task shards x{world}",
                       "l2": "inputs larger than L2 (D/J/K 3 x %.0f MB + device pair data), no flush" % (n * n * 8 / 1e6),
                       "pair_build_s": pair_s},
            "s_per_iter": ms * 1e-3,
            "quartets_per_s": stats["quartets"] / (ms * 1e-3),
            "gpu_launches": int(launches_per_build * args.steps),
            "clocks": clk, "roofline": roof,
            "e2e": {"value": flops_total / (ms_e2e * 1e-3) / 1e12, "unit": UNIT, "ms_per_step": ms_e2e,
                    "h2d_bytes_per_step": int(n * n * 8), "d2h_bytes_per_step": int(2 * n * n * 8)}}
    if mixed is not None:
        line["mixed_precision"] = mixed
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(sh, Dh, args.tau, flops_total, target_s=args.cpu_seconds)
    if args.class_times and rank == 0:
        line["class_ms"] = {f"({names[int((math.isqrt(8*i+1)-1)//2)]}|"
                            f"{names[i - int((math.isqrt(8*i+1)-1)//2) * (int((math.isqrt(8*i+1)-1)//2) + 1) // 2]})":
                            [round(float(cls_ms[i] / max(cls_n[i], 1)), 4), float(cls_flops[i]), int(cls_q[i]),
                             int(P.last_prim_quartets[i])]
                            for i in range(len(cls_ms)) if cls_n[i] > 0}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["mako", "reference"], default="mako")
    ap.add_argument("--config", default=DEFAULT_CONFIG, choices=sorted(mi.CONFIGS))
    ap.add_argument("--tau", type=float, default=TAU)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    # both CPU legs size their quartet sample with the same target, so their extrapolations agree
    ap.add_argument("--cpu-seconds", type=float, default=8.0)
    ap.add_argument("--ref-step-s", type=float, default=8.0)
    ap.add_argument("--class-times", action="store_true")
    ap.add_argument("--mixed", type=float, default=1e-6,
                    help="thresh_fp64 of the reduced-precision measurement (0 = skip)")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    return run_mako(args)


if __name__ == "__main__":
    sys.exit(main())

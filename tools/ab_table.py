"""Per-class A/B table of round-2 kernel experiments (bench.py --class-times lines under profiles/ab_r02/):
    python tools/ab_table.py > profiles/bench_r02_ab.md"""
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
RUNS = [("r2b_nostrip", "round-1 kernels (interleaved shards)"), ("r2b_strip", "+ K-row strips (lane-per-ket)"),
        ("r2b_swap", "+ strips, 25 classes transposed"), ("r2c_rb", "+ strips, batched R (L <= 7)"),
        ("r2d_rbswap", "+ strips, batched R + transposed"), ("r2e_rb2", "no strips, batched R (L <= 6) incl. (pp|pp) ... (dp|ds) moved to family 4"),
        ("r2e_rb2s", "r2e_rb2 + (ds|pp) (dp|pp) (dp|ds) transposed"), ("r2f_main", "picks + flipped K atomics + staged lane-per-ket atomics"),
        ("r2g_main", "picks + bra-row K atomics + staged lane-per-ket atomics"), ("r2i_nostage", "r2g_main without staging"),
        ("r2i_main", "r2g_main + fragment-order E~ (DMMA operands)"),
        ("r2j_main", "r2i_main without staging, GEMM2 k-steps interleaved over accumulators"),
        ("r2k_main", "r2j_main (repeat)"), ("r2k_nob", "r2k_main with row-major GEMM2 B operands"),
        ("r2k_rbg", "r2k_main + batched R for L >= 7 with lane-group recursion (not kept)")]
# session 3: band/shell pair order with K_ac/K_bc run aggregation (S6, tools/exp/r2_band_order.patch)
RUNS2 = [("r2n_pre", "fec4888 kernels (reference for this group)"),
         ("r2m_allband_dmma", "all buckets in band order; run aggregation in every family (lane-per-ket, ket-first, DMMA)"),
         ("r2m_q0_dmma", "the same kernels on the Q order (no runs)"),
         ("r2o_allband", "all buckets in band order; aggregation in lane-per-ket + ket-first (values first, then the scan)"),
         ("r2o_q0", "the same kernels on the Q order"),
         ("r2p_allband_kfold", "all buckets in band order; aggregation in lane-per-ket only"),
         ("r2q_tpqperm", "Q order storage, lane-per-ket classes walk a band permutation; aggregation in lane-per-ket"),
         ("r2q_q0", "the same kernels on the Q order")]
# session 3: super-batched R phase of the slot-batched kernel, and more classes on that kernel
RUNS3 = [("r2r_pre", "fec4888 kernels (reference for this group)"),
         ("r2r_superbatch", "slot-batched (dp|pp): R rows of RCAP / K_AB slots per R phase, one primitive quartet per lane (kept)"),
         ("r2r_slab2", "+ (pp|pp) (fs|pp) (fs|dp) (fp|pp) on the slot-batched kernel"),
         ("r2r_slab3", "ket-first classes (dp|ds) (fs|ds) (fp|ps) (fd|ps) (ds|pp) on the slot-batched kernel; (dp|ps) falls to lane-per-ket")]
# session 3: per-class family re-selection from all-on / all-off runs
RUNS4 = [("r2s_main", "picks of 82991a3"),
         ("r2s_tpqx", "every lane-per-ket-eligible light-ket class on the lane-per-ket kernel"),
         ("r2s_swapall", "every warp-per-quartet class transposed"), ("r2s_swapnone", "no class transposed"),
         ("r2s_kfnsa", "no ket-first kernel, warp-per-quartet classes transposed"),
         ("r2s_kfnsn", "no ket-first kernel, nothing transposed")]
# session 3: per-class occupancy caps
RUNS5 = [("r2v_main", "main (tpq kernels compiled with __launch_bounds__(128, 1): the ss-ket classes slower, reverted)"),
         ("r2v_caps", "(ps|ps) at 5 CTAs/SM; ket-first (dp|ds) (fd|ps) (dd|ps) (fs|ds) at 3 CTAs/SM: only (dd|ps) kept"),
         ("r2x_main", "lane-per-ket kernel refactored into free / capped instantiations, no caps"),
         ("r2x_tpqcap3", "lane-per-ket (pp|ps) (ds|ps) (fs|ps) at 3 CTAs/SM (168 registers, 64-324 B spills): kept"),
         ("r2x_tpqcap4", "(ds|ps) (fs|ps) at 4 CTAs/SM, (pp|ps) at 3: slower"),
         ("r2y_main", "main with the lane-per-ket caps (ef7f4a2)"),
         ("r2z_jkcap", "every warp-per-quartet class at 4 CTAs/SM: kept for (fd|dp) (ff|pp) (ff|fs)"),
         ("r2z_jknocap", "no warp-per-quartet class capped: kept for (fd|fd)"),
         ("r2f2_main", "main with the re-selected caps (015c565)"),
         ("r2sw_rball", "batched lane-per-quartet R for every warp-per-quartet class with L <= 6: kept for (fp|ds)"),
         ("r2sw_rbnone", "batched R for none"),
         ("r2sw_fball", "GEMM2 B operands from the fragment-order copy for every class"),
         ("r2sw_fbnone", "... for none (row-major E~)"),
         ("r2f3_main", "final kernels (076314d)"),
         ("r2kc_kfnocap", "no 3-CTA register cap on any ket-first class: every cap of the list still pays ((ds|pp) 551 -> 637 ms without)")]
d = {}
for name, _ in RUNS + RUNS2 + RUNS3 + RUNS4 + RUNS5:
    p = os.path.join(ROOT, "profiles", "ab_r02", name + ".jsonl")
    if os.path.exists(p):
        d[name] = json.loads(open(p).read())
names = [n for n, _ in RUNS if n in d]
print("# Round-2 kernel experiments, per class (valinomycin-sized def2-TZVP build, ms per class kernel)\n")
print("Each column is one `bench.py --class-times` run on a B200 (`tools/exp/r2_*.sh`); the build total is the")
print("first row.  Lower is better.\n")
for n, desc in RUNS:
    if n in d:
        print(f"- `{n}`: {desc}")
print()
print("| class | " + " | ".join(names) + " |")
print("|---|" + "---|" * len(names))
print("| **build s** | " + " | ".join("%.3f" % d[n]["s_per_iter"] for n in names) + " |")
classes = list(d[names[0]]["class_ms"])
classes.sort(key=lambda k: -d[names[0]]["class_ms"][k][0])
for k in classes:
    print(f"| {k} | " + " | ".join("%.1f" % d[n]["class_ms"][k][0] if k in d[n]["class_ms"] else "" for n in names) + " |")

names2 = [n for n, _ in RUNS2 if n in d]
if names2:
    print("\n## Band/shell pair order and K_ac/K_bc run aggregation (session 3; not kept)\n")
    for n, desc in RUNS2:
        if n in d:
            print(f"- `{n}`: {desc}")
    print()
    print("| class | " + " | ".join(names2) + " |")
    print("|---|" + "---|" * len(names2))
    print("| **build s** | " + " | ".join("%.3f" % d[n]["s_per_iter"] for n in names2) + " |")
    for k in classes:
        print(f"| {k} | " + " | ".join("%.1f" % d[n]["class_ms"][k][0] if k in d[n]["class_ms"] else "" for n in names2) + " |")

names3 = [n for n, _ in RUNS3 if n in d]
if names3:
    print("\n## Slot-batched kernel with a super-batched R phase (session 3)\n")
    for n, desc in RUNS3:
        if n in d:
            print(f"- `{n}`: {desc}")
    print()
    print("| class | " + " | ".join(names3) + " |")
    print("|---|" + "---|" * len(names3))
    print("| **build s** | " + " | ".join("%.3f" % d[n]["s_per_iter"] for n in names3) + " |")
    for k in classes:
        print(f"| {k} | " + " | ".join("%.1f" % d[n]["class_ms"][k][0] if k in d[n]["class_ms"] else "" for n in names3) + " |")

names4 = [n for n, _ in RUNS4 if n in d]
if names4:
    print("\n## Per-class family re-selection (session 3): (dp|ps) -> lane-per-ket, (ff|dd) (ff|fd) transposed\n")
    for n, desc in RUNS4:
        if n in d:
            print(f"- `{n}`: {desc}")
    print()
    print("| class | " + " | ".join(names4) + " |")
    print("|---|" + "---|" * len(names4))
    print("| **build s** | " + " | ".join("%.3f" % d[n]["s_per_iter"] for n in names4) + " |")
    for k in classes:
        print(f"| {k} | " + " | ".join("%.1f" % d[n]["class_ms"][k][0] if k in d[n]["class_ms"] else "" for n in names4) + " |")

names5 = [n for n, _ in RUNS5 if n in d]
if names5:
    print("\n## Occupancy caps per class (session 3)\n")
    for n, desc in RUNS5:
        if n in d:
            print(f"- `{n}`: {desc}")
    print()
    print("| class | " + " | ".join(names5) + " |")
    print("|---|" + "---|" * len(names5))
    print("| **build s** | " + " | ".join("%.3f" % d[n]["s_per_iter"] for n in names5) + " |")
    for k in classes:
        print(f"| {k} | " + " | ".join("%.1f" % d[n]["class_ms"][k][0] if k in d[n]["class_ms"] else "" for n in names5) + " |")

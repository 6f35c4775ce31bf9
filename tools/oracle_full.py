"""Check of the cpu_baseline extrapolation: the full oracle J/K build of a config timed
directly, next to the quartet-sample estimate bench.py's cpu_baseline leg makes in the same process.

    python tools/oracle_full.py --config gly10-ccpvtz > profiles/oracle_full_r02.json

Calls only oracle/ (test infrastructure: orc_schwarz, orc_jk, orc_jk_qsample) on the seeded synthetic
density of the config; the GPU path is not involved.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
import mako_inputs as mi  # noqa: E402
import oracle  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="gly10-ccpvtz")
    ap.add_argument("--tau", type=float, default=bench.TAU)
    ap.add_argument("--sample-s", type=float, default=8.0)
    a = ap.parse_args()
    mol, basis = mi.config_molecule(a.config)
    sh = mi.shells_for(mol, basis)
    D = mi.synthetic_density(sh.nbf(), mol.nelec // 2, seed=0)
    Q = oracle.schwarz(sh)
    flops, nq = bench.workload_flops(sh, Q, a.tau)
    S, ovh = bench.oracle_sample_seconds(sh, D, a.tau, Q, a.sample_s)
    S = max(S, 2)
    ts, est = bench.oracle_sampled_build(sh, D, a.tau, Q, S, S // 2, ovh)
    t0 = time.perf_counter()
    oracle.jk(sh, D, a.tau, Q=Q)
    full = time.perf_counter() - t0
    print(json.dumps({"config": a.config, "nbf": sh.nbf(), "tau": a.tau, "quartets": nq, "gemm_flops": flops,
                      "threads": oracle.num_threads(), "full_build_s": full,
                      "full_build_tflops": flops / full / 1e12,
                      "sample": {"S": S, "sample_s": ts, "overhead_s": ovh, "estimate_s": est,
                                 "estimate_over_full": est / full}}))


if __name__ == "__main__":
    main()

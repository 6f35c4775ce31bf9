"""Write oracle J/K blocks of sampled shell pairs for a large config to tests/golden/ (test fixture).

    python tools/make_golden_blocks.py --config ubiquitin-def2tzvp --npairs 8 --seed 0

Calls only oracle/ (orc_schwarz, orc_jk_blocks: the definition-level blocks J_{mn} = sum (mn|ls) D_ls,
K_{ml} = sum (mn|ls) D_ns with the Schwarz rule Q_ab Q_cd >= tau, Eq. 1, north_star)
on the seeded synthetic density of the config (mako_inputs.synthetic_density, seed 0).  The GPU test
tests/test_gpu_c5.py rebuilds the same D and compares its full build's blocks with these.
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import mako_inputs as mi  # noqa: E402
import oracle  # noqa: E402


def pick_pairs(sh, n, seed):
    """Same-atom pairs of mixed l (non-trivial J and K), neighbour-atom pairs, one distant pair."""
    rng = np.random.default_rng(seed)
    atoms = np.unique(sh.atom)
    heavy = [a for a in atoms if (sh.l[sh.atom == a] == 3).any()]
    out = []
    for a in rng.choice(heavy, n // 2, replace=False):
        idx = np.nonzero(sh.atom == a)[0]
        x, y = rng.choice(idx, 2, replace=False)
        out.append((int(max(x, y)), int(min(x, y))))
    xyz = sh.xyz
    while len(out) < n - 1:
        x = int(rng.integers(sh.nshell))
        d = np.sqrt(((xyz - xyz[x]) ** 2).sum(1))
        near = np.nonzero((d > 0.5) & (d < 5.0))[0]
        if len(near):
            out.append((x, int(rng.choice(near))))
    x = int(rng.integers(sh.nshell))
    d = np.sqrt(((xyz - xyz[x]) ** 2).sum(1))
    out.append((x, int(np.argmax(d))))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="ubiquitin-def2tzvp")
    ap.add_argument("--npairs", type=int, default=8)
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--tau", type=float, default=1e-12)
    a = ap.parse_args()
    mol, basis = mi.config_molecule(a.config)
    sh = mi.shells_for(mol, basis)
    n = sh.nbf()
    t0 = time.time()
    D = mi.synthetic_density(n, mol.nelec // 2, seed=0)
    t1 = time.time()
    Q = oracle.schwarz(sh)
    t2 = time.time()
    pairs = pick_pairs(sh, a.npairs, a.seed)
    Jb, Kb = oracle.jk_blocks(sh, D, pairs, tau=a.tau, Q=Q)
    t3 = time.time()
    out = os.path.join(ROOT, "tests", "golden", f"{a.config}_blocks.npz")
    np.savez_compressed(out, pairs=np.array(pairs, np.int32), J=np.concatenate([j.ravel() for j in Jb]),
                        K=np.concatenate([k.ravel() for k in Kb]), tau=a.tau, nbf=n, nshell=sh.nshell)
    meta = {"config": a.config, "basis": mi.basis_label(basis), "nbf": n, "nshell": sh.nshell, "tau": a.tau,
            "density": "mako_inputs.synthetic_density(nbf, nelec // 2, seed=0)", "pairs": pairs,
            "oracle": "orc_schwarz + orc_jk_blocks (oracle/mako_oracle.c), definition-level J/K blocks",
            "cite": "PAPER.md:L106-L109 (Eq. 1); J/K definitions of BASELINE.json north_star",
            "seconds": {"density": t1 - t0, "schwarz": t2 - t1, "blocks": t3 - t2},
            "threads": oracle.num_threads()}
    json.dump(meta, open(out[:-4] + ".json", "w"), indent=1)
    print(json.dumps(meta))


if __name__ == "__main__":
    main()

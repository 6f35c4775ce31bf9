"""Pins for the oracle ERIs (Eq. 1-2): closed forms, mpmath brute force,
invariants.  None of these retype the oracle's Obara-Saika/HGP recurrences.
"""
import math

import mpmath as mp
import numpy as np
import pytest

import oracle
from mako_inputs import Shells

mp.mp.dps = 30


def single_prim_shells(specs):
    """specs: list of (l, alpha, center xyz) -> Shells of single-primitive shells (coef 1)."""
    l = np.array([s[0] for s in specs], np.int32)
    return Shells(np.arange(len(specs), dtype=np.int32), l, np.ones(len(specs), np.int32),
                  np.array([s[2] for s in specs], np.float64), np.array([s[1] for s in specs], np.float64),
                  np.ones(len(specs)))


def ssss_closed(a, A, b, B, c, C, d, D):
    """Closed-form (ss|ss) for unnormalised primitives (Boys 1950 / Szabo-Ostlund A.41) in mpmath."""
    p, q = a + b, c + d
    AB2 = sum((A[i] - B[i]) ** 2 for i in range(3))
    CD2 = sum((C[i] - D[i]) ** 2 for i in range(3))
    P = [(a * A[i] + b * B[i]) / p for i in range(3)]
    Q = [(c * C[i] + d * D[i]) / q for i in range(3)]
    PQ2 = sum((P[i] - Q[i]) ** 2 for i in range(3))
    T = p * q / (p + q) * PQ2
    F0 = mp.mpf(1) if T == 0 else mp.sqrt(mp.pi / T) * mp.erf(mp.sqrt(T)) / 2
    return 2 * mp.pi ** mp.mpf(2.5) / (p * q * mp.sqrt(p + q)) * mp.exp(-a * b / p * AB2 - c * d / q * CD2) * F0


def norm2_mp(alpha, powers):
    """<g|g> of x^i y^j z^k exp(-alpha r^2) by mpmath quadrature (independent of any closed form)."""
    r = mp.mpf(1)
    for n in powers:
        r *= mp.quad(lambda x: x ** (2 * n) * mp.exp(-2 * alpha * x * x), [-mp.inf, mp.inf])
    return r


def cart_eri_mp(exps, centers, powers):
    """Primitive Cartesian ERI via center derivatives of the closed-form (ss|ss):
    u^1 g = D g/(2a), u^2 g = D^2 g/(4a^2) + g/(2a), u^3 g = D^3 g/(8a^3) + 3 D g/(4a^2),
    u^4 g = D^4 g/(16a^4) + 3 D^2 g/(4a^3) + 3 g/(4a^2),  D = d/dA_x acting on exp(-a (x-A_x)^2)."""
    a = [mp.mpf(e) for e in exps]
    X0 = [mp.mpf(v) for c in centers for v in c]

    # expansion of u^n g into derivative orders: list of (order, coefficient) per (center, axis)
    def expand(n, al):
        if n == 0:
            return [(0, mp.mpf(1))]
        if n == 1:
            return [(1, 1 / (2 * al))]
        if n == 2:
            return [(2, 1 / (4 * al ** 2)), (0, 1 / (2 * al))]
        if n == 3:
            return [(3, 1 / (8 * al ** 3)), (1, 3 / (4 * al ** 2))]
        if n == 4:  # D^4 g = 16a^4 u^4 g - 48a^3 u^2 g + 12a^2 g
            return [(4, 1 / (16 * al ** 4)), (2, 3 / (4 * al ** 3)), (0, 3 / (4 * al ** 2))]
        raise ValueError

    terms = [((), mp.mpf(1))]
    for ci in range(4):
        for ax in range(3):
            new = []
            for orders, cf in terms:
                for o, c2 in expand(powers[ci][ax], a[ci]):
                    new.append((orders + (o,), cf * c2))
            terms = new

    def f(*x):
        C = [x[3 * i:3 * i + 3] for i in range(4)]
        return ssss_closed(a[0], C[0], a[1], C[1], a[2], C[2], a[3], C[3])

    total = mp.mpf(0)
    for orders, cf in terms:
        if sum(orders) == 0:
            total += cf * f(*X0)
        else:
            total += cf * mp.diff(f, X0, orders)
    return total


def test_ssss_closed_form_contracted():
    # contracted s shells on three centers, normalised primitive coefficients as tabulated
    sh = Shells(np.arange(3, dtype=np.int32), np.zeros(3, np.int32), np.array([3, 2, 1], np.int32),
                np.array([[0, 0, 0], [0.3, -1.2, 0.7], [1.9, 0.4, -0.5]], np.float64),
                np.array([3.0, 0.8, 0.2, 1.5, 0.4, 0.6]), np.array([0.2, 0.5, 0.4, 0.6, 0.5, 1.0]))
    poff = [0, 3, 5, 6]
    # contracted normalisation computed here from the closed-form s overlap (pi/(a+b))^{3/2}
    def nrm(s):
        e = sh.exps[poff[s]:poff[s + 1]]; c = sh.coefs[poff[s]:poff[s + 1]]
        cn = c * (2 * e / math.pi) ** 0.75
        S = sum(cn[i] * cn[j] * (math.pi / (e[i] + e[j])) ** 1.5 for i in range(len(e)) for j in range(len(e)))
        return e, cn / math.sqrt(S)
    for (A, B, C, D) in [(0, 1, 2, 0), (1, 1, 2, 2), (2, 0, 1, 1), (0, 0, 0, 0)]:
        ref = mp.mpf(0)
        ea, ca = nrm(A); eb, cb = nrm(B); ec, cc = nrm(C); ed, cd = nrm(D)
        for i in range(len(ea)):
            for j in range(len(eb)):
                for k in range(len(ec)):
                    for m in range(len(ed)):
                        ref += ca[i] * cb[j] * cc[k] * cd[m] * ssss_closed(
                            mp.mpf(ea[i]), [mp.mpf(v) for v in sh.xyz[A]], mp.mpf(eb[j]), [mp.mpf(v) for v in sh.xyz[B]],
                            mp.mpf(ec[k]), [mp.mpf(v) for v in sh.xyz[C]], mp.mpf(ed[m]), [mp.mpf(v) for v in sh.xyz[D]])
        got = oracle.eri_quartet(sh, A, B, C, D)[0, 0, 0, 0]
        assert abs(got - float(ref)) < 1e-14 * abs(float(ref))


CASES = [
    # (l list, exps, centers, powers per center, cart component index per shell)
    ((2, 1, 0, 0), (1.3, 0.7, 0.9, 0.4),
     ((0.0, 0.1, -0.2), (0.8, -0.4, 0.3), (-0.5, 0.9, 0.6), (0.2, 0.3, 1.1)),
     ((2, 0, 0), (0, 1, 0), (0, 0, 0), (0, 0, 0))),
    ((1, 0, 1, 0), (0.9, 1.6, 0.5, 2.1),
     ((0.1, 0.0, 0.0), (0.0, 0.7, -0.3), (1.0, -0.2, 0.4), (-0.6, 0.5, 0.0)),
     ((1, 0, 0), (0, 0, 0), (0, 0, 1), (0, 0, 0))),
    ((2, 2, 1, 0), (0.8, 1.1, 0.6, 0.9),
     ((0.0, 0.0, 0.0), (0.5, 0.4, -0.3), (-0.4, 0.6, 0.8), (0.9, -0.7, 0.2)),
     ((1, 1, 0), (0, 1, 1), (1, 0, 0), (0, 0, 0))),
    ((3, 0, 1, 1), (0.7, 1.2, 0.8, 0.5),
     ((0.2, -0.1, 0.0), (-0.6, 0.3, 0.5), (0.4, 0.8, -0.7), (0.0, -0.5, 0.6)),
     ((1, 2, 0), (0, 0, 0), (0, 1, 0), (0, 0, 1))),
    ((0, 0, 3, 2), (1.0, 0.6, 0.9, 1.4),
     ((0.0, 0.0, 0.3), (0.7, 0.1, -0.2), (-0.3, 0.5, 0.4), (0.5, -0.6, 0.9)),
     ((0, 0, 0), (0, 0, 0), (0, 0, 3), (1, 0, 1))),
    # g functions (row f3): (g_xxyz s | p_x s) and (s s | g_zzzz s)
    ((4, 0, 1, 0), (0.9, 1.3, 0.7, 0.6),
     ((0.1, -0.2, 0.3), (-0.7, 0.4, 0.2), (0.5, 0.6, -0.4), (0.3, -0.5, 0.8)),
     ((2, 1, 1), (0, 0, 0), (1, 0, 0), (0, 0, 0))),
    ((0, 0, 4, 0), (1.1, 0.8, 0.6, 1.5),
     ((0.0, 0.2, -0.1), (0.6, -0.3, 0.4), (-0.4, 0.1, 0.7), (0.2, 0.9, -0.5)),
     ((0, 0, 0), (0, 0, 0), (0, 0, 4), (0, 0, 0))),
]


def _cidx(x, y, z):
    l = x + y + z
    return (l - x) * (l - x + 1) // 2 + (l - x - y)


@pytest.mark.parametrize("case", range(len(CASES)))
def test_cartesian_eri_vs_mpmath_derivatives(case):
    ls, exps, centers, powers = CASES[case]
    sh = single_prim_shells([(ls[i], exps[i], centers[i]) for i in range(4)])
    blk = oracle.eri_quartet(sh, 0, 1, 2, 3, pure=False)
    idx = tuple(_cidx(*powers[i]) for i in range(4))
    raw = cart_eri_mp(exps, centers, powers)
    nrm = mp.mpf(1)
    for i in range(4):
        # normalisation of the x^l component (the Cartesian convention of include/mako.h)
        nrm *= norm2_mp(mp.mpf(exps[i]), (ls[i], 0, 0))
    ref = float(raw / mp.sqrt(nrm))
    assert abs(blk[idx] - ref) <= 1e-13 * abs(ref) + 1e-16, (blk[idx], ref)


def _random_basis(seed, lmax=3, n=4):
    rng = np.random.default_rng(seed)
    specs = []
    ls, nps, xyz, ex, cf = [], [], [], [], []
    for i in range(n):
        l = int(rng.integers(0, lmax + 1)); k = int(rng.integers(1, 3))
        ls.append(l); nps.append(k); xyz.append(rng.uniform(-1.0, 1.0, 3))
        ex += list(np.exp(rng.uniform(np.log(0.3), np.log(4.0), k))); cf += list(rng.uniform(0.3, 1.0, k))
    return Shells(np.arange(n, dtype=np.int32), np.array(ls, np.int32), np.array(nps, np.int32),
                  np.array(xyz), np.array(ex), np.array(cf))


def _fixed_basis():
    return Shells(np.arange(5, dtype=np.int32), np.array([3, 2, 1, 0, 2], np.int32), np.array([1, 2, 1, 2, 1], np.int32),
                  np.array([[0, 0, 0], [0.9, 0.2, -0.4], [-0.3, 1.1, 0.5], [0.4, -0.8, 0.9], [0.0, 0.0, 0.0]]),
                  np.array([0.9, 1.7, 0.5, 1.2, 3.0, 0.4, 0.7]), np.array([1.0, 0.6, 0.5, 1.0, 0.4, 0.7, 1.0]))


@pytest.mark.parametrize("pure", [True, False])
def test_eightfold_symmetry_psd_schwarz(pure):
    sh = _fixed_basis()
    eri = oracle.eri_full(sh, pure=pure)
    for perm in ["jikl", "ijlk", "jilk", "klij", "lkij", "klji", "lkji"]:
        assert np.allclose(eri, np.einsum("ijkl->" + perm, eri), rtol=0, atol=1e-14)
    N = eri.shape[0]
    M = eri.reshape(N * N, N * N)
    w = np.linalg.eigvalsh(M)
    assert w.min() >= -1e-12 * w.max()
    Q = oracle.schwarz(sh, pure=pure)
    # Cauchy-Schwarz between shell blocks
    off = np.concatenate([[0], np.cumsum([(2 * l + 1) if pure else (l + 1) * (l + 2) // 2 for l in sh.l])])
    for a in range(sh.nshell):
        for b in range(sh.nshell):
            for c in range(sh.nshell):
                for d in range(sh.nshell):
                    blk = eri[off[a]:off[a + 1], off[b]:off[b + 1], off[c]:off[c + 1], off[d]:off[d + 1]]
                    assert np.abs(blk).max() <= Q[a, b] * Q[c, d] * (1 + 1e-12)


@pytest.mark.parametrize("pure", [True, False])
def test_schwarz_is_sqrt_of_max_diagonal(pure):
    """orc_schwarz pinned EXACTLY to its definition (DESIGN reading R6):
    Q_ab = sqrt(max_{m in a, n in b} |(mn|mn)|) from the full ERI tensor -- a Q taken over all block
    (mm|nn) or a sum of the diagonal would fail here (it is only an upper bound in the test above).  The
    maximum over the whole (ab|ab) block equals the diagonal maximum (Cauchy-Schwarz), so that reading
    is the same definition."""
    for sh in (_fixed_basis(), _random_basis(4), _random_basis(9)):
        eri = oracle.eri_full(sh, pure=pure)
        Q = oracle.schwarz(sh, pure=pure)
        off = np.concatenate([[0], np.cumsum([(2 * l + 1) if pure else (l + 1) * (l + 2) // 2 for l in sh.l])])
        wrong = 0
        for a in range(sh.nshell):
            for b in range(sh.nshell):
                diag = [abs(eri[m, n, m, n]) for m in range(off[a], off[a + 1]) for n in range(off[b], off[b + 1])]
                ref = np.sqrt(max(diag))
                assert abs(Q[a, b] - ref) <= 1e-14 * ref, (a, b, Q[a, b], ref)
                blk = eri[off[a]:off[a + 1], off[b]:off[b + 1], off[a]:off[a + 1], off[b]:off[b + 1]]
                assert abs(np.sqrt(np.abs(blk).max()) - ref) <= 1e-14 * ref
                mmnn = [abs(eri[m, m, n, n]) for m in range(off[a], off[a + 1]) for n in range(off[b], off[b + 1])]
                wrong = max(wrong, abs(np.sqrt(max(mmnn)) - ref) / ref)
        assert wrong > 1e-3  # the (mm|nn) reading differs: the pin discriminates


def test_spherical_orthonormal_and_known_forms():
    for l in range(5):
        C = oracle.sph_coeffs(l)
        # Cartesian metric of normalised x^l-convention functions (same exponent/centre), by mpmath quad
        cart = [(x, y, l - x - y) for x in range(l, -1, -1) for y in range(l - x, -1, -1)]
        G = np.zeros((len(cart), len(cart)))
        n_l = norm2_mp(mp.mpf(1), (l, 0, 0))
        for i, a in enumerate(cart):
            for j, b in enumerate(cart):
                v = mp.mpf(1)
                for k in range(3):
                    s = a[k] + b[k]
                    v *= mp.quad(lambda x: x ** s * mp.exp(-2 * x * x), [-mp.inf, mp.inf])
                G[i, j] = float(v / n_l)
        assert np.allclose(C @ G @ C.T, np.eye(2 * l + 1), atol=1e-13)
    # p is (x, y, z); d0 = zz - xx/2 - yy/2 on x^l-normalised Cartesians (real solid harmonic 3z^2 - r^2)
    assert np.allclose(oracle.sph_coeffs(1), np.eye(3))
    d = oracle.sph_coeffs(2)
    assert np.allclose(d[2], [-0.5, 0, 0, -0.5, 0, 1.0], atol=1e-15)
    # d_xy, d_yz, d_xz, d_{x2-y2}: positive leading coefficients on xy, yz, xz, xx
    assert d[0, 1] > 0 and d[1, 4] > 0 and d[3, 2] > 0 and d[4, 0] > 0 and abs(d[4, 0] + d[4, 3]) < 1e-15
    f = oracle.sph_coeffs(3)
    # f_{z^3} (m=0) ~ z(2z^2 - 3x^2 - 3y^2): ratios zzz : xxz : yyz
    r = f[3]
    ic = {c: i for i, c in enumerate([(x, y, 3 - x - y) for x in range(3, -1, -1) for y in range(3 - x, -1, -1)])}
    # all Cartesians share the x^l normalisation, so coefficients are proportional to the polynomial's
    assert r[ic[(0, 0, 3)]] > 0
    assert abs(r[ic[(2, 0, 1)]] / r[ic[(0, 0, 3)]] + 1.5) < 1e-14
    assert abs(r[ic[(0, 2, 1)]] / r[ic[(0, 0, 3)]] + 1.5) < 1e-14
    # f_{x(x^2-3y^2)} (m=3): xxx : xyy = 1 : -3 ; f_{y(3x^2-y^2)} (m=-3): xxy : yyy = 3 : -1
    assert abs(f[6][ic[(1, 2, 0)]] / f[6][ic[(3, 0, 0)]] + 3.0) < 1e-14 and f[6][ic[(3, 0, 0)]] > 0
    assert abs(f[0][ic[(0, 3, 0)]] / f[0][ic[(2, 1, 0)]] + 1.0 / 3.0) < 1e-14 and f[0][ic[(2, 1, 0)]] > 0


def _rotation(seed):
    rng = np.random.default_rng(seed)
    q, r = np.linalg.qr(rng.standard_normal((3, 3)))
    return q * np.sign(np.linalg.det(q))


def test_addition_theorem_rotation_invariance():
    """sum_m phi_lm(r)^2 is rotation invariant, so sum_{m,m'} (a_m a_m | b_m' b_m') is invariant under a
    rigid rotation of all centres.  A wrong spherical coefficient breaks this."""
    base = [(2, 0.8, (0.0, 0.0, 0.0)), (3, 0.6, (0.9, -0.4, 0.5)), (1, 1.1, (-0.7, 0.3, 0.8))]
    def inv(specs):
        sh = single_prim_shells(specs)
        b = oracle.eri_quartet(sh, 0, 0, 1, 1)
        c = oracle.eri_quartet(sh, 0, 1, 0, 1)
        e = oracle.eri_quartet(sh, 0, 2, 1, 2)
        # traces over the rotating index pairs and a Frobenius norm: all orthogonal invariants
        return (np.einsum("iijj->", b), np.einsum("ijij->", c), np.sum(e ** 2))
    v0 = inv(base)
    R = _rotation(3)
    v1 = inv([(l, a, tuple(R @ np.array(c))) for (l, a, c) in base])
    assert np.allclose(v0, v1, rtol=1e-12, atol=1e-15)


def test_pure_equals_cart_for_l_le_1():
    sh = Shells(np.arange(3, dtype=np.int32), np.array([1, 0, 1], np.int32), np.array([2, 1, 1], np.int32),
                np.array([[0, 0, 0], [0.5, 0.5, -0.2], [-0.4, 0.9, 0.3]]), np.array([1.1, 0.3, 0.7, 0.5]),
                np.array([0.5, 0.6, 1.0, 1.0]))
    a = oracle.eri_full(sh, pure=True)
    b = oracle.eri_full(sh, pure=False)
    assert np.array_equal(a, b)

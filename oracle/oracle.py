"""ctypes binding of oracle/liboracle.so (plain C, OpenMP).  TEST INFRASTRUCTURE ONLY."""
import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "mako_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

_dp = ctypes.POINTER(ctypes.c_double)
_ip = ctypes.POINTER(ctypes.c_int)


def build_oracle(force=False):
    """Compile the oracle with gcc (-O2 -fopenmp).  Building the checker is not using it."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", _LIB, _SRC, "-lm"])
    return _LIB


def _get():
    global _lib
    if _lib is None:
        build_oracle()
        _lib = ctypes.CDLL(_LIB)
    return _lib


def _d(a):
    return a.ctypes.data_as(_dp)


def _i(a):
    return a.ctypes.data_as(_ip)


def _basis_args(sh, pure):
    l = np.ascontiguousarray(sh.l, dtype=np.int32)
    npr = np.ascontiguousarray(sh.nprim, dtype=np.int32)
    xyz = np.ascontiguousarray(sh.xyz, dtype=np.float64)
    ex = np.ascontiguousarray(sh.exps, dtype=np.float64)
    cf = np.ascontiguousarray(sh.coefs, dtype=np.float64)
    keep = (l, npr, xyz, ex, cf)
    return keep, (ctypes.c_int(len(l)), _i(l), _i(npr), _d(xyz), _d(ex), _d(cf), ctypes.c_int(1 if pure else 0))


def _nf(l, pure):
    return 2 * l + 1 if pure else (l + 1) * (l + 2) // 2


def _check(rc, what):
    if rc != 0:
        raise RuntimeError(f"oracle {what} failed with status {rc}")


def num_threads():
    return _get().orc_num_threads()


def boys(mmax, T):
    out = np.zeros(mmax + 1)
    _check(_get().orc_boys(ctypes.c_int(mmax), ctypes.c_double(T), _d(out)), "boys")
    return out


def sph_coeffs(l):
    out = np.zeros((2 * l + 1, (l + 1) * (l + 2) // 2))
    _check(_get().orc_sph_coeffs(ctypes.c_int(l), _d(out)), "sph_coeffs")
    return out


def eri_quartet(sh, a, b, c, d, pure=True):
    keep, args = _basis_args(sh, pure)
    shp = tuple(_nf(int(sh.l[s]), pure) for s in (a, b, c, d))
    out = np.zeros(shp)
    _check(_get().orc_eri_quartet(*args, a, b, c, d, _d(out)), "eri_quartet")
    return out


def eri_full(sh, pure=True):
    keep, args = _basis_args(sh, pure)
    N = sh.nbf(pure)
    out = np.zeros((N, N, N, N))
    _check(_get().orc_eri_full(*args, _d(out)), "eri_full")
    return out


def schwarz(sh, pure=True):
    keep, args = _basis_args(sh, pure)
    Q = np.zeros((sh.nshell, sh.nshell))
    _check(_get().orc_schwarz(*args, _d(Q)), "schwarz")
    return Q


def jk(sh, D, tau=0.0, shard=0, nshards=1, pure=True, Q=None):
    keep, args = _basis_args(sh, pure)
    N = sh.nbf(pure)
    D = np.ascontiguousarray(D, dtype=np.float64)
    assert D.shape == (N, N)
    J = np.zeros((N, N)); K = np.zeros((N, N))
    Qp = None
    if Q is not None:
        Q = np.ascontiguousarray(Q, dtype=np.float64)
        Qp = _d(Q)
    _check(_get().orc_jk(*args, _d(D), ctypes.c_double(tau), shard, nshards, Qp, _d(J), _d(K)), "jk")
    return J, K


def jk_qsample(sh, D, tau, shard, nshards, pure=True, Q=None):
    """J/K over the canonical quartets (P, R) with (P(P+1)/2 + R) % nshards == shard (orc_jk_qsample): a
    uniform 1/nshards sample of every class for timing the oracle on large builds; shards sum to jk()."""
    keep, args = _basis_args(sh, pure)
    N = sh.nbf(pure)
    D = np.ascontiguousarray(D, dtype=np.float64)
    J = np.zeros((N, N)); K = np.zeros((N, N))
    Qp = None
    if Q is not None:
        Q = np.ascontiguousarray(Q, dtype=np.float64)
        Qp = _d(Q)
    _check(_get().orc_jk_qsample(*args, _d(D), ctypes.c_double(tau), ctypes.c_longlong(shard),
                                 ctypes.c_longlong(nshards), Qp, _d(J), _d(K)), "jk_qsample")
    return J, K


def jk_dw(sh, D, tau, tau_dw, pure=True, Q=None):
    """J/K with the Schwarz rule at tau plus density-weighted screening at tau_dw (orc_jk_dw)."""
    keep, args = _basis_args(sh, pure)
    N = sh.nbf(pure)
    D = np.ascontiguousarray(D, dtype=np.float64)
    assert D.shape == (N, N)
    J = np.zeros((N, N)); K = np.zeros((N, N))
    Qp = None
    if Q is not None:
        Q = np.ascontiguousarray(Q, dtype=np.float64)
        Qp = _d(Q)
    _check(_get().orc_jk_dw(*args, _d(D), ctypes.c_double(tau), ctypes.c_double(tau_dw), Qp, _d(J), _d(K)), "jk_dw")
    return J, K


def jk_blocks(sh, D, pairs, tau=0.0, Q=None, pure=True):
    """Exact J/K blocks for shell pairs [(x, y), ...]: returns lists of [n_x, n_y] arrays."""
    keep, args = _basis_args(sh, pure)
    D = np.ascontiguousarray(D, dtype=np.float64)
    pairs = np.ascontiguousarray(np.asarray(pairs, dtype=np.int32).reshape(-1, 2))
    sizes = [_nf(int(sh.l[x]), pure) * _nf(int(sh.l[y]), pure) for x, y in pairs]
    Jb = np.zeros(sum(sizes)); Kb = np.zeros(sum(sizes))
    Qp = None
    if Q is not None:
        Q = np.ascontiguousarray(Q, dtype=np.float64)
        Qp = _d(Q)
    _check(_get().orc_jk_blocks(*args, _d(D), ctypes.c_double(tau), Qp, len(pairs), _i(pairs), _d(Jb), _d(Kb)),
           "jk_blocks")
    Js, Ks, o = [], [], 0
    for (x, y), s in zip(pairs, sizes):
        shp = (_nf(int(sh.l[x]), pure), _nf(int(sh.l[y]), pure))
        Js.append(Jb[o:o + s].reshape(shp)); Ks.append(Kb[o:o + s].reshape(shp)); o += s
    return Js, Ks


def one_electron(sh, mol, pure=True):
    keep, args = _basis_args(sh, pure)
    N = sh.nbf(pure)
    Z = np.ascontiguousarray(mol.Z, dtype=np.float64)
    axyz = np.ascontiguousarray(mol.xyz_bohr, dtype=np.float64)
    S = np.zeros((N, N)); T = np.zeros((N, N)); V = np.zeros((N, N))
    _check(_get().orc_one_electron(*args, mol.natm, _d(Z), _d(axyz), _d(S), _d(T), _d(V)), "one_electron")
    return S, T, V


def nuclear_repulsion(mol):
    """E_nuc = sum_{A<B} Z_A Z_B / R_AB."""
    Z = mol.Z.astype(np.float64)
    x = mol.xyz_bohr
    e = 0.0
    for i in range(mol.natm):
        for j in range(i):
            e += Z[i] * Z[j] / np.linalg.norm(x[i] - x[j])
    return e

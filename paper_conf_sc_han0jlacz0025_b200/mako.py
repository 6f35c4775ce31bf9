"""Python API over the C ABI (include/mako.h): Basis, Pairs, build_jk, eri_batch, boys.

PyTorch provides device memory and streams only; every step of the J/K path runs in libmako's
CUDA kernels.  Device tensors must be float64, contiguous, on the handle's CUDA device.
"""
import ctypes

import numpy as np
import torch

from . import _lib
from ._lib import check


def _i32(a):
    a = np.ascontiguousarray(a, dtype=np.int32)
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_int))


def _f64(a):
    a = np.ascontiguousarray(a, dtype=np.float64)
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def _stream_ptr(stream):
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _dev_ptr(t, name):
    if not (isinstance(t, torch.Tensor) and t.is_cuda and t.dtype == torch.float64 and t.is_contiguous()):
        raise ValueError(f"{name} must be a contiguous float64 CUDA tensor")
    return ctypes.c_void_p(t.data_ptr())


class Basis:
    """Gaussian basis on a molecule.  ``shells`` is a mako_inputs.Shells-like
    object (atom, l, nprim, exps, coefs); ``Z``/``xyz`` the atoms (bohr)."""

    def __init__(self, Z, xyz, shells, pure=True):
        self._lib = _lib.load()
        Zc, Zp = _i32(Z)
        Xc, Xp = _f64(np.asarray(xyz).reshape(-1))
        a, ap = _i32(shells.atom)
        l, lp = _i32(shells.l)
        n, npp = _i32(shells.nprim)
        e, ep = _f64(shells.exps)
        c, cp = _f64(shells.coefs)
        h = ctypes.c_void_p()
        check(self._lib.mako_basis_create(len(Zc), Zp, Xp, len(l), ap, lp, npp, ep, cp, 1 if pure else 0,
                                          ctypes.byref(h)))
        self.handle = h
        nbf = ctypes.c_int()
        check(self._lib.mako_basis_nbf(h, ctypes.byref(nbf)))
        self.nbf = nbf.value
        self.nshell = len(l)
        ao = np.zeros(self.nshell + 1, np.int32)
        check(self._lib.mako_basis_ao_offsets(h, ao.ctypes.data_as(ctypes.POINTER(ctypes.c_int))))
        self.ao_offsets = ao
        self.l = l.copy()

    @classmethod
    def from_molecule(cls, mol, shells):
        return cls(mol.Z, mol.xyz_bohr, shells)

    def close(self):
        if getattr(self, "handle", None):
            self._lib.mako_basis_destroy(self.handle)
            self.handle = None

    __del__ = close


class Pairs:
    """Screened shell-pair data (Schwarz threshold tau), device resident."""

    def __init__(self, basis, tau=1e-12, stream=None):
        self._lib = basis._lib
        self.basis = basis  # keeps the basis alive
        self.tau = tau
        h = ctypes.c_void_p()
        check(self._lib.mako_shellpairs_screen(basis.handle, float(tau), _stream_ptr(stream), ctypes.byref(h)))
        self.handle = h
        self.device = torch.device("cuda", torch.cuda.current_device())

    def stats(self, thresh=None):
        a, b, c = ctypes.c_longlong(), ctypes.c_longlong(), ctypes.c_longlong()
        check(self._lib.mako_pairs_stats(self.handle, float(self.tau if thresh is None else thresh), ctypes.byref(a),
                                         ctypes.byref(b), ctypes.byref(c)))
        return {"pairs": a.value, "prim_pairs": b.value, "quartets": c.value}

    def flops(self, thresh=None, shard=0, nshards=1):
        f, q, pq = ctypes.c_double(), ctypes.c_longlong(), ctypes.c_longlong()
        check(self._lib.mako_pairs_flops(self.handle, float(self.tau if thresh is None else thresh), shard, nshards,
                                         ctypes.byref(f), ctypes.byref(q), ctypes.byref(pq)))
        return {"gemm_flops": f.value, "quartets": q.value, "prim_quartets": pq.value}

    def launches(self, thresh=None, shard=0, nshards=1):
        n = ctypes.c_int()
        check(self._lib.mako_build_jk_launches(self.handle, float(self.tau if thresh is None else thresh), shard,
                                               nshards, ctypes.byref(n)))
        return n.value

    def class_flops(self, thresh=None, shard=0, nshards=1):
        f = np.zeros(_lib.NCLASS)
        q = np.zeros(_lib.NCLASS, np.int64)
        pq = np.zeros(_lib.NCLASS, np.int64)
        llp = lambda x: x.ctypes.data_as(ctypes.POINTER(ctypes.c_longlong))
        check(self._lib.mako_pairs_class_flops(self.handle, float(self.tau if thresh is None else thresh), shard,
                                               nshards, f.ctypes.data_as(ctypes.POINTER(ctypes.c_double)), llp(q),
                                               llp(pq)))
        self.last_prim_quartets = pq
        return f, q

    def profile(self, enable=True):
        check(self._lib.mako_profile_enable(self.handle, 1 if enable else 0))

    def profile_read(self):
        ms = np.zeros(_lib.NCLASS)
        n = np.zeros(_lib.NCLASS, np.int64)
        check(self._lib.mako_profile_read(self.handle, ms.ctypes.data_as(ctypes.POINTER(ctypes.c_double)),
                                          n.ctypes.data_as(ctypes.POINTER(ctypes.c_longlong))))
        return ms, n

    def close(self):
        if getattr(self, "handle", None):
            self._lib.mako_pairs_destroy(self.handle)
            self.handle = None

    __del__ = close


MAKO_JK_DENSITY_SCREEN = 1
MAKO_JK_ACCUMULATE = 2
MAKO_ERI_REDUCED = 1


def density_delta(pairs, D, D_prev, dD=None, stream=None):
    """dD = D - D_prev on the device and max|dD| (mako_density_delta; synchronises `stream`)."""
    if dD is None:
        dD = torch.empty_like(D)
    n = pairs.basis.nbf
    for name, t in (("D", D), ("D_prev", D_prev), ("dD", dD)):
        if not isinstance(t, torch.Tensor) or tuple(t.shape) != (n, n):
            raise ValueError(f"{name} must be a {n}x{n} tensor")
    m = ctypes.c_double()
    check(pairs._lib.mako_density_delta(pairs.handle, _dev_ptr(D, "D"), _dev_ptr(D_prev, "D_prev"), _dev_ptr(dD, "dD"),
                                        ctypes.byref(m), _stream_ptr(stream)))
    return dD, m.value


def build_jk(pairs, D, thresh=None, J=None, K=None, shard=0, nshards=1, stream=None, density_screen=False,
             thresh_fp64=None, accumulate=False):
    """J_{mn} = sum (mn|ls) D_ls, K_{ml} = sum (mn|ls) D_ns on the GPU (north_star).  Async on `stream`
    (density_screen=True: mako_build_jk_ex with MAKO_JK_DENSITY_SCREEN, which synchronises `stream`).
    thresh_fp64: stage-aware reduced-precision build (mako_build_jk_mixed; synchronises `stream`):
    quartets whose contribution bound Q_ab Q_cd max|D| is below ~thresh_fp64 run the TF32 tier.
    accumulate=True: J += J[D], K += K[D] (MAKO_JK_ACCUMULATE; J and K must be given)."""
    if accumulate and (J is None or K is None):
        raise ValueError("accumulate=True needs the J and K to accumulate into")
    n = pairs.basis.nbf
    if J is None:
        J = torch.empty_like(D)
    if K is None:
        K = torch.empty_like(D)
    # the C ABI takes raw pointers: check shapes and devices here so that an undersized or foreign
    # buffer is rejected instead of written past its end
    dev = getattr(pairs, "device", None)
    for name, t in (("D", D), ("J", J), ("K", K)):
        if not isinstance(t, torch.Tensor) or tuple(t.shape) != (n, n):
            raise ValueError(f"{name} must be a {n}x{n} tensor")
        if dev is not None and t.device != dev:
            raise ValueError(f"{name} is on {t.device}, the pairs live on {dev}")
    t = float(pairs.tau if thresh is None else thresh)
    flags = (MAKO_JK_DENSITY_SCREEN if density_screen else 0) | (MAKO_JK_ACCUMULATE if accumulate else 0)
    if thresh_fp64 is not None:
        check(pairs._lib.mako_build_jk_mixed(pairs.handle, _dev_ptr(D, "D"), t, float(thresh_fp64), flags,
                                             _dev_ptr(J, "J"), _dev_ptr(K, "K"), int(shard), int(nshards),
                                             _stream_ptr(stream)))
    elif flags:
        check(pairs._lib.mako_build_jk_ex(pairs.handle, _dev_ptr(D, "D"), t, flags, _dev_ptr(J, "J"),
                                          _dev_ptr(K, "K"), int(shard), int(nshards), _stream_ptr(stream)))
    else:
        check(pairs._lib.mako_build_jk(pairs.handle, _dev_ptr(D, "D"), t, _dev_ptr(J, "J"), _dev_ptr(K, "K"),
                                       int(shard), int(nshards), _stream_ptr(stream)))
    return J, K


def class_reduced():
    """[MAKO_NCLASS] bool: classes with a reduced-precision (TF32) kernel (mako_class_reduced)."""
    m = np.zeros(_lib.NCLASS, np.int32)
    check(_lib.load().mako_class_reduced(m.ctypes.data_as(ctypes.POINTER(ctypes.c_int))))
    return m.astype(bool)


FAMILY_KERNELS = {0: "tpq_jk_kernel", 1: "kf_jk_kernel", 2: "kf_jk_kernel (transposed)", 3: "slab_jk_kernel",
                  4: "jk_kernel", 5: "jk_kernel (transposed)"}


def class_family():
    """[MAKO_NCLASS] int: kernel family per class (mako_class_family; FAMILY_KERNELS names them)."""
    m = np.zeros(_lib.NCLASS, np.int32)
    check(_lib.load().mako_class_family(m.ctypes.data_as(ctypes.POINTER(ctypes.c_int))))
    return m


def eri_batch(basis, quartets, stream=None, device=None, reduced=False):
    """Shell-quartet ERI blocks (test entry).  Returns a list of numpy-shaped torch tensors on the GPU.
    reduced=True: mako_eri_batch_ex with MAKO_ERI_REDUCED (the TF32 tier where the class has one)."""
    q, qp = _i32(np.asarray(quartets).reshape(-1, 4))
    # out-of-range shells are left to the C ABI to reject (MAKO_ERR_INVALID)
    nf = lambda s: 2 * int(basis.l[s]) + 1 if 0 <= s < basis.nshell else 0
    sizes = [int(np.prod([nf(s) for s in row])) for row in q]
    out = torch.empty(sum(sizes), dtype=torch.float64, device=device or "cuda")
    check(basis._lib.mako_eri_batch_ex(basis.handle, len(q), qp, _dev_ptr(out, "out"), out.numel(),
                                       MAKO_ERI_REDUCED if reduced else 0, _stream_ptr(stream)))
    res, o = [], 0
    for row, s in zip(q, sizes):
        res.append(out[o:o + s].view(*[2 * basis.l[x] + 1 for x in row]))
        o += s
    return res


def boys(T, mmax, stream=None):
    """Device Boys evaluator of the hot path: T (CUDA float64 [n]) -> [n, mmax+1]."""
    lib = _lib.load()
    T = T.contiguous()
    out = torch.empty((T.numel(), mmax + 1), dtype=torch.float64, device=T.device)
    check(lib.mako_boys(T.numel(), _dev_ptr(T, "T"), int(mmax), _dev_ptr(out, "out"), _stream_ptr(stream)))
    return out

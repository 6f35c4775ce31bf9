"""CPU-side checks of the C-ABI boundary: libmako.so loads, exports every symbol include/mako.h
declares, and compute entry points fail loudly (MAKO_ERR_CUDA) without a GPU -- no CPU fallback."""
import ctypes
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _header_functions():
    src = open(os.path.join(ROOT, "include", "mako.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(mako_[a-z_0-9]+)\s*\(", src)))


def test_header_lists_boundary():
    fns = _header_functions()
    for f in ["mako_basis_create", "mako_shellpairs_screen", "mako_build_jk", "mako_eri_batch"]:
        assert f in fns


def test_library_exports_every_header_symbol():
    from paper_conf_sc_han0jlacz0025_b200 import _lib
    lib = _lib.load()
    for f in _header_functions():
        assert hasattr(lib, f), f
    assert sorted(_lib.EXPORTS) == _header_functions()
    assert b"sm_100a" in lib.mako_version()


def _sass(function):
    """SASS of one kernel of the library (cuobjdump -fun; the whole 60+ MB dump takes a minute)."""
    import subprocess
    from paper_conf_sc_han0jlacz0025_b200 import _lib
    return subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", "-fun", function, _lib.LIB_PATH],
                          capture_output=True, text=True).stdout


def test_library_is_sm100a_cubin():
    import subprocess
    from paper_conf_sc_han0jlacz0025_b200 import _lib
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", _lib.LIB_PATH], capture_output=True, text=True)
    assert "sm_100a" in out.stdout
    # FP64 tensor-core MMA (mma.sync .f64) in the (ff|ff) class kernel
    assert "DMMA" in _sass("_ZN4mako14jk_kernel_freeILi9ELi9ELb0EEEvNS_6JKArgsE")


def test_errors_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("CPU-only check")
    from paper_conf_sc_han0jlacz0025_b200 import _lib
    lib = _lib.load()
    h = ctypes.c_void_p()
    Z = np.array([1, 1], np.int32)
    xyz = np.array([0, 0, 0, 0, 0, 1.4])
    l = np.array([0, 0], np.int32)
    npr = np.array([1, 1], np.int32)
    at = np.array([0, 1], np.int32)
    e = np.array([1.0, 1.0])
    c = np.array([1.0, 1.0])
    ip = lambda a: a.ctypes.data_as(ctypes.POINTER(ctypes.c_int))
    dp = lambda a: a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))
    st = lib.mako_basis_create(2, ip(Z), dp(xyz), 2, ip(at), ip(l), ip(npr), dp(e), dp(c), 1, ctypes.byref(h))
    assert st == 3 and b"no CUDA device" in lib.mako_last_error()
    # argument validation happens before device checks
    st = lib.mako_basis_create(2, ip(Z), dp(xyz), 2, ip(at), ip(l), ip(npr), dp(e), dp(c), 0, ctypes.byref(h))
    assert st == 2
    assert lib.mako_build_jk(None, None, 0.0, None, None, 0, 1, None) == 1


def test_reduced_precision_tier_boundary():
    """the TF32 tier exists in the library (SASS HMMA.1688.F32.TF32 next to DMMA), covers
    every high-l class with l <= 3 (L >= 8, where the basis transformation dominates), and the mixed build
    validates its arguments before touching the device."""
    from paper_conf_sc_han0jlacz0025_b200 import _lib, class_reduced
    assert "HMMA.1688.F32.TF32" in _sass("_ZN4mako11jk_kernel_qILi9ELi9ELb0EEEvNS_6JKArgsE")
    assert "HMMA.1688.F32.TF32" in _sass("_ZN4mako11jk_kernel_qILi8ELi8ELb0EEEvNS_6JKArgsE")  # (fd|fd)
    m = class_reduced()
    bl = [(la, lb) for la in range(5) for lb in range(la + 1)]
    for X in range(15):
        for Y in range(X + 1):
            if sum(bl[X]) + sum(bl[Y]) >= 8 and max(bl[X] + bl[Y]) <= 3:
                assert m[X * (X + 1) // 2 + Y], (bl[X], bl[Y])
    assert not m[0] and not m[1]  # (ss|ss), (ps|ss): lane-per-ket FP64 only
    lib = _lib.load()
    assert lib.mako_build_jk_mixed(None, None, 0.0, 1e-6, 0, None, None, 0, 1, None) == 1
    assert lib.mako_class_reduced(None) == 1

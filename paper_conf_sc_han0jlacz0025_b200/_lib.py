"""ctypes binding of libmako.so (include/mako.h).  Argument marshalling only.

The library is built in-tree by ``python -m paper_conf_sc_han0jlacz0025_b200.build`` (or
``__graft_entry__.build()``).  There is no fallback: if libmako.so is missing this module raises.
"""
import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libmako.so")
# experiments only: MAKO_LIB names an alternative in-tree build (build.py --variant NAME -> libmako_NAME.so)
if os.environ.get("MAKO_LIB"):
    LIB_PATH = os.path.join(HERE, "libmako_%s.so" % os.environ["MAKO_LIB"])

MAKO_OK = 0
NCLASS = 120  # MAKO_NCLASS (l <= 4: 15 pair buckets)
STATUS = {0: "MAKO_OK", 1: "MAKO_ERR_INVALID", 2: "MAKO_ERR_UNSUPPORTED", 3: "MAKO_ERR_CUDA", 4: "MAKO_ERR_OOM",
          5: "MAKO_ERR_STATE"}

# every symbol include/mako.h declares (checked by tests/test_abi.py)
EXPORTS = ["mako_basis_create", "mako_basis_nbf", "mako_basis_nshell", "mako_basis_ao_offsets", "mako_basis_destroy",
           "mako_shellpairs_screen", "mako_pairs_stats", "mako_pairs_flops", "mako_pairs_destroy", "mako_build_jk",
           "mako_build_jk_launches", "mako_eri_batch", "mako_boys", "mako_last_error", "mako_version",
           "mako_pairs_class_flops", "mako_profile_enable", "mako_profile_read", "mako_build_jk_ex",
           "mako_build_jk_mixed", "mako_class_reduced", "mako_eri_batch_ex", "mako_class_family",
           "mako_density_delta"]


class MakoError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


_lib = None
_ip = ctypes.POINTER(ctypes.c_int)
_dp = ctypes.POINTER(ctypes.c_double)
_vp = ctypes.c_void_p
_ll = ctypes.c_longlong


def load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not found: build it with `python -m paper_conf_sc_han0jlacz0025_b200.build` "
                          "(there is no CPU fallback)")
    lib = ctypes.CDLL(LIB_PATH)
    sig = {
        "mako_basis_create": ([ctypes.c_int, _ip, _dp, ctypes.c_int, _ip, _ip, _ip, _dp, _dp, ctypes.c_int,
                               ctypes.POINTER(_vp)], ctypes.c_int),
        "mako_basis_nbf": ([_vp, _ip], ctypes.c_int),
        "mako_basis_nshell": ([_vp, _ip], ctypes.c_int),
        "mako_basis_ao_offsets": ([_vp, _ip], ctypes.c_int),
        "mako_basis_destroy": ([_vp], None),
        "mako_shellpairs_screen": ([_vp, ctypes.c_double, _vp, ctypes.POINTER(_vp)], ctypes.c_int),
        "mako_pairs_stats": ([_vp, ctypes.c_double, ctypes.POINTER(_ll), ctypes.POINTER(_ll), ctypes.POINTER(_ll)],
                             ctypes.c_int),
        "mako_pairs_flops": ([_vp, ctypes.c_double, ctypes.c_int, ctypes.c_int, _dp, ctypes.POINTER(_ll),
                              ctypes.POINTER(_ll)], ctypes.c_int),
        "mako_pairs_destroy": ([_vp], None),
        "mako_build_jk": ([_vp, _vp, ctypes.c_double, _vp, _vp, ctypes.c_int, ctypes.c_int, _vp], ctypes.c_int),
        "mako_build_jk_ex": ([_vp, _vp, ctypes.c_double, ctypes.c_uint, _vp, _vp, ctypes.c_int, ctypes.c_int, _vp],
                             ctypes.c_int),
        "mako_build_jk_mixed": ([_vp, _vp, ctypes.c_double, ctypes.c_double, ctypes.c_uint, _vp, _vp, ctypes.c_int,
                                 ctypes.c_int, _vp], ctypes.c_int),
        "mako_density_delta": ([_vp, _vp, _vp, _vp, _dp, _vp], ctypes.c_int),
        "mako_class_reduced": ([_ip], ctypes.c_int),
        "mako_class_family": ([_ip], ctypes.c_int),
        "mako_eri_batch_ex": ([_vp, ctypes.c_int, _ip, _vp, ctypes.c_size_t, ctypes.c_uint, _vp], ctypes.c_int),
        "mako_build_jk_launches": ([_vp, ctypes.c_double, ctypes.c_int, ctypes.c_int, _ip], ctypes.c_int),
        "mako_eri_batch": ([_vp, ctypes.c_int, _ip, _vp, ctypes.c_size_t, _vp], ctypes.c_int),
        "mako_boys": ([ctypes.c_int, _vp, ctypes.c_int, _vp, _vp], ctypes.c_int),
        "mako_pairs_class_flops": ([_vp, ctypes.c_double, ctypes.c_int, ctypes.c_int, _dp, ctypes.POINTER(_ll),
                                    ctypes.POINTER(_ll)], ctypes.c_int),
        "mako_profile_enable": ([_vp, ctypes.c_int], ctypes.c_int),
        "mako_profile_read": ([_vp, _dp, ctypes.POINTER(_ll)], ctypes.c_int),
        "mako_last_error": ([], ctypes.c_char_p),
        "mako_version": ([], ctypes.c_char_p),
    }
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    _lib = lib
    return lib


def check(status):
    if status != MAKO_OK:
        msg = load().mako_last_error()
        raise MakoError(status, msg.decode() if msg else "")

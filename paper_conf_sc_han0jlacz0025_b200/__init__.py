"""B200-native direct-SCF J/K build (Mako, SC'25 hot path) -- see DESIGN.md and include/mako.h."""
from ._lib import LIB_PATH, MakoError, EXPORTS

__all__ = ["LIB_PATH", "MakoError", "EXPORTS", "Basis", "Pairs", "build_jk", "eri_batch", "boys", "class_reduced", "density_delta",
           "IncrementalJK"]


def __getattr__(name):
    if name in ("Basis", "Pairs", "build_jk", "eri_batch", "boys", "class_reduced", "density_delta"):
        from . import mako
        return getattr(mako, name)
    if name == "IncrementalJK":
        from .incremental import IncrementalJK
        return IncrementalJK
    raise AttributeError(name)

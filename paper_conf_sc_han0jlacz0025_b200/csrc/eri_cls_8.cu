// eri_cls_8.cu -- kernel instantiations for bra bucket 8 (generated layout; see eri_kernels.cuh)
#define MAKO_DEFINE_KERNELS
#include "eri_kernels.cuh"

MAKO_INSTANTIATE(8, 0)
MAKO_INSTANTIATE(8, 1)
MAKO_INSTANTIATE(8, 2)
MAKO_INSTANTIATE(8, 3)
MAKO_INSTANTIATE(8, 4)
MAKO_INSTANTIATE(8, 5)
MAKO_INSTANTIATE(8, 6)
MAKO_INSTANTIATE(8, 7)
MAKO_INSTANTIATE(8, 8)

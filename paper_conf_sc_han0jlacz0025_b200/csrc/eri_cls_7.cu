// eri_cls_7.cu -- kernel instantiations for bra bucket 7 (generated layout; see eri_kernels.cuh)
#define MAKO_DEFINE_KERNELS
#include "eri_kernels.cuh"

MAKO_INSTANTIATE(7, 0)
MAKO_INSTANTIATE(7, 1)
MAKO_INSTANTIATE(7, 2)
MAKO_INSTANTIATE(7, 3)
MAKO_INSTANTIATE(7, 4)
MAKO_INSTANTIATE(7, 5)
MAKO_INSTANTIATE(7, 6)
MAKO_INSTANTIATE(7, 7)

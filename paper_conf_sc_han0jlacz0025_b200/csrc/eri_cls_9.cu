// eri_cls_9.cu -- kernel instantiations for bra bucket 9 (generated layout; see eri_kernels.cuh)
#define MAKO_DEFINE_KERNELS
#include "eri_kernels.cuh"

MAKO_INSTANTIATE(9, 0)
MAKO_INSTANTIATE(9, 1)
MAKO_INSTANTIATE(9, 2)
MAKO_INSTANTIATE(9, 3)
MAKO_INSTANTIATE(9, 4)
MAKO_INSTANTIATE(9, 5)
MAKO_INSTANTIATE(9, 6)
MAKO_INSTANTIATE(9, 7)
MAKO_INSTANTIATE(9, 8)
MAKO_INSTANTIATE(9, 9)

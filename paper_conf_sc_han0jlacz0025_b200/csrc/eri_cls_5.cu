// eri_cls_5.cu -- kernel instantiations for bra bucket 5 (generated layout; see eri_kernels.cuh)
#define MAKO_DEFINE_KERNELS
#include "eri_kernels.cuh"

MAKO_INSTANTIATE(5, 0)
MAKO_INSTANTIATE(5, 1)
MAKO_INSTANTIATE(5, 2)
MAKO_INSTANTIATE(5, 3)
MAKO_INSTANTIATE(5, 4)
MAKO_INSTANTIATE(5, 5)

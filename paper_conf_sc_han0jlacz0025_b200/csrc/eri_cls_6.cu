// eri_cls_6.cu -- kernel instantiations for bra bucket 6 (generated layout; see eri_kernels.cuh)
#define MAKO_DEFINE_KERNELS
#include "eri_kernels.cuh"

MAKO_INSTANTIATE(6, 0)
MAKO_INSTANTIATE(6, 1)
MAKO_INSTANTIATE(6, 2)
MAKO_INSTANTIATE(6, 3)
MAKO_INSTANTIATE(6, 4)
MAKO_INSTANTIATE(6, 5)
MAKO_INSTANTIATE(6, 6)

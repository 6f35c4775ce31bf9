// eri_cls_4.cu -- kernel instantiations for bra bucket 4 (generated layout; see eri_kernels.cuh)
#define MAKO_DEFINE_KERNELS
#include "eri_kernels.cuh"

MAKO_INSTANTIATE(4, 0)
MAKO_INSTANTIATE(4, 1)
MAKO_INSTANTIATE(4, 2)
MAKO_INSTANTIATE(4, 3)
MAKO_INSTANTIATE(4, 4)

// eri_cls_3.cu -- kernel instantiations for bra bucket 3 (generated layout; see eri_kernels.cuh)
#define MAKO_DEFINE_KERNELS
#include "eri_kernels.cuh"

MAKO_INSTANTIATE(3, 0)
MAKO_INSTANTIATE(3, 1)
MAKO_INSTANTIATE(3, 2)
MAKO_INSTANTIATE(3, 3)

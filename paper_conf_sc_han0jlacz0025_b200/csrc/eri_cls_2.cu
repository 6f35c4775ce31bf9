// eri_cls_2.cu -- kernel instantiations for bra bucket 2 (generated layout; see eri_kernels.cuh)
#define MAKO_DEFINE_KERNELS
#include "eri_kernels.cuh"

MAKO_INSTANTIATE(2, 0)
MAKO_INSTANTIATE(2, 1)
MAKO_INSTANTIATE(2, 2)

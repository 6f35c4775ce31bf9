// eri_cls_1.cu -- kernel instantiations for bra bucket 1 (generated layout; see eri_kernels.cuh)
#define MAKO_DEFINE_KERNELS
#include "eri_kernels.cuh"

MAKO_INSTANTIATE(1, 0)
MAKO_INSTANTIATE(1, 1)

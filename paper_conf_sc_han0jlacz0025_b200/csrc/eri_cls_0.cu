// eri_cls_0.cu -- kernel instantiations for bra bucket 0 (generated layout; see eri_kernels.cuh)
#define MAKO_DEFINE_KERNELS
#include "eri_kernels.cuh"

MAKO_INSTANTIATE(0, 0)

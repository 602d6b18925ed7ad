// conv_r3_cm1.cu — radius-3 TMA convolution kernels, column mode COL_CLAMP (see conv_impl.cuh).
#include "conv_impl.cuh"

namespace mapsm {
MAPSM_CONV_BIG_INST(, 3, kConvNS<3>, COL_CLAMP)
}  // namespace mapsm

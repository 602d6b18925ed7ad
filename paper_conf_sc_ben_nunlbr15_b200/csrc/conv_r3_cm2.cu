// conv_r3_cm2.cu — radius-3 TMA convolution kernels, column mode COL_ZERO (see conv_impl.cuh).
#include "conv_impl.cuh"

namespace mapsm {
MAPSM_CONV_BIG_INST(, 3, kConvNS<3>, COL_ZERO)
}  // namespace mapsm

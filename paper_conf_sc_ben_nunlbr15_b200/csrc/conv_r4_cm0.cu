// conv_r4_cm0.cu — radius-4 TMA convolution kernels, column mode COL_WRAP (see conv_impl.cuh).
#include "conv_impl.cuh"

namespace mapsm {
MAPSM_CONV_BIG_INST(, 4, kConvNS<4>, COL_WRAP)
}  // namespace mapsm

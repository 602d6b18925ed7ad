// conv_r3_cm0.cu — radius-3 TMA convolution kernels, column mode COL_WRAP (see conv_impl.cuh).
#include "conv_impl.cuh"

namespace mapsm {
MAPSM_CONV_BIG_INST(, 3, kConvNS<3>, COL_WRAP)
}  // namespace mapsm

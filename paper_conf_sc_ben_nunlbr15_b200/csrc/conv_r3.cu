// conv_r3.cu — radius-3 instantiation of the fp32 window convolution (see conv_impl.cuh);
// the TMA kernels themselves are compiled in conv_r3_cm0.cu .. conv_r3_cm2.cu.
#include "conv_impl.cuh"

namespace mapsm {
MAPSM_CONV_BIG_INST_ALL(extern, 3, kConvNS<3>)
template cudaError_t launch_conv_radius<3>(const StencilGeom&, const RowBands&, const float*, int, cudaStream_t,
                                               const FusedLink*);
}  // namespace mapsm

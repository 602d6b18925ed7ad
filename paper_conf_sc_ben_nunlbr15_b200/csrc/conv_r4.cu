// conv_r4.cu — radius-4 instantiation of the fp32 window convolution (see conv_impl.cuh);
// the TMA kernels themselves are compiled in conv_r4_cm0.cu .. conv_r4_cm2.cu.
#include "conv_impl.cuh"

namespace mapsm {
MAPSM_CONV_BIG_INST_ALL(extern, 4, kConvNS<4>)
template cudaError_t launch_conv_radius<4>(const StencilGeom&, const RowBands&, const float*, int, cudaStream_t,
                                               const FusedLink*);
}  // namespace mapsm

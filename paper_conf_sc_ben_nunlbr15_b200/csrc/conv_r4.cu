// conv_r4.cu — radius-4 instantiation of the fp32 window convolution (see conv_impl.cuh).
#include "conv_impl.cuh"

namespace mapsm {
template cudaError_t launch_conv_radius<4>(const StencilGeom&, const RowBands&, const float*, int, cudaStream_t,
                                               const FusedLink*);
}  // namespace mapsm

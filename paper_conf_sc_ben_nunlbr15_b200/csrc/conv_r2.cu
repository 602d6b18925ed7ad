// conv_r2.cu — radius-2 instantiation of the fp32 window convolution (see conv_impl.cuh).
#include "conv_impl.cuh"

namespace mapsm {
template cudaError_t launch_conv_radius<2>(const StencilGeom&, const RowBands&, const float*, int, cudaStream_t,
                                               const FusedLink*);
}  // namespace mapsm

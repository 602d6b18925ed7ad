// conv_r1.cu — radius-1 instantiation of the fp32 window convolution (see conv_impl.cuh).
#include "conv_impl.cuh"

namespace mapsm {
template cudaError_t launch_conv_radius<1>(const StencilGeom&, const RowBands&, const float*, int, cudaStream_t,
                                               const FusedLink*);
}  // namespace mapsm

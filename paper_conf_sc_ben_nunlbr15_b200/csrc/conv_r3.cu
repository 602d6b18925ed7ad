// conv_r3.cu — radius-3 instantiation of the fp32 window convolution (see conv_impl.cuh);
// the TMA kernels themselves are compiled in conv_r3_cm0.cu .. conv_r3_cm2.cu.
#include "conv_impl.cuh"

namespace mapsm {
MAPSM_CONV_BIG_INST_ALL(extern, 3, kConvNS<3>)
template cudaError_t launch_conv_radius<3>(const StencilGeom&, const RowBands&, const float*, int, cudaStream_t,
                                               const FusedLink*);
cudaError_t conv_upload_weights_r3(int cm, int slot, const float* w) {
    switch (cm) {
        case COL_WRAP: return conv_detail::conv_upload_weights_t<3, COL_WRAP>(slot, w);
        case COL_CLAMP: return conv_detail::conv_upload_weights_t<3, COL_CLAMP>(slot, w);
        default: return conv_detail::conv_upload_weights_t<3, COL_ZERO>(slot, w);
    }
}
}  // namespace mapsm

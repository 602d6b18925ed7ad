// conv_r4.cu — radius-4 instantiation of the fp32 window convolution (see conv_impl.cuh);
// the TMA kernels themselves are compiled in conv_r4_cm0.cu .. conv_r4_cm2.cu.
#include "conv_impl.cuh"

namespace mapsm {
MAPSM_CONV_BIG_INST_ALL(extern, 4, kConvNS<4>)
template cudaError_t launch_conv_radius<4>(const StencilGeom&, const RowBands&, const float*, int, cudaStream_t,
                                               const FusedLink*);
cudaError_t conv_upload_weights_r4(int cm, int slot, const float* w) {
    switch (cm) {
        case COL_WRAP: return conv_detail::conv_upload_weights_t<4, COL_WRAP>(slot, w);
        case COL_CLAMP: return conv_detail::conv_upload_weights_t<4, COL_CLAMP>(slot, w);
        default: return conv_detail::conv_upload_weights_t<4, COL_ZERO>(slot, w);
    }
}
}  // namespace mapsm

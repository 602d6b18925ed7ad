// conv_r2.cu — radius-2 instantiation of the fp32 window convolution (see conv_impl.cuh).
#include "conv_impl.cuh"

namespace mapsm {
template cudaError_t launch_conv_radius<2>(const StencilGeom&, const RowBands&, const float*, int, cudaStream_t,
                                               const FusedLink*);
cudaError_t conv_upload_weights_r2(int cm, int slot, const float* w) {
    if (2 < conv_detail::kConvPairMinR) return cudaSuccess;
    switch (cm) {
        case COL_WRAP: return conv_detail::conv_upload_weights_t<2, COL_WRAP>(slot, w);
        case COL_CLAMP: return conv_detail::conv_upload_weights_t<2, COL_CLAMP>(slot, w);
        default: return conv_detail::conv_upload_weights_t<2, COL_ZERO>(slot, w);
    }
}
bool conv_uses_weight_slot(int r) { return r >= conv_detail::kConvPairMinR && r <= 4; }
}  // namespace mapsm

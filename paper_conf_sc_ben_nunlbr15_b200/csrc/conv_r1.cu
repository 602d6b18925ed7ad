// conv_r1.cu — radius-1 instantiation of the fp32 window convolution (see conv_impl.cuh).
#include "conv_impl.cuh"
#include "conv_tb.cuh"

namespace mapsm {
template cudaError_t launch_conv_radius<1>(const StencilGeom&, const RowBands&, const float*, int, cudaStream_t,
                                               const FusedLink*);
cudaError_t conv_upload_weights_r1(int cm, int slot, const float* w) {
    const cudaError_t e = conv_detail::tb2_upload_weights<1>(slot, w);  // two-generation kernel's pairs
    if (e != cudaSuccess) return e;
    switch (cm) {
        case COL_WRAP: return conv_detail::conv_upload_weights_t<1, COL_WRAP>(slot, w);
        case COL_CLAMP: return conv_detail::conv_upload_weights_t<1, COL_CLAMP>(slot, w);
        default: return conv_detail::conv_upload_weights_t<1, COL_ZERO>(slot, w);
    }
}
cudaError_t launch_conv_tb2_r1(const StencilGeom& g, const RowBands& b, int zt, int zb, int num_sms, cudaStream_t s) {
    return conv_detail::launch_conv_tb2_r<1>(g, b, zt, zb, num_sms, s);
}
}  // namespace mapsm

// conv.cu — radius dispatch of the fp32 window convolution (kernels in
// conv_impl.cuh, one translation unit per radius: conv_r1.cu .. conv_r4.cu;
// radii 5..8 in conv_wide.cu).
#include <cuda_runtime.h>
#include <stdlib.h>

#include "kernels.h"

namespace mapsm {

template <int R>
cudaError_t launch_conv_radius(const StencilGeom& g, const RowBands& b, const float* weights, int num_sms,
                               cudaStream_t s, const FusedLink* link);

cudaError_t conv_upload_weights_r1(int cm, int slot, const float* w);
cudaError_t conv_upload_weights_r2(int cm, int slot, const float* w);
cudaError_t launch_conv_tb2_r1(const StencilGeom& g, const RowBands& b, int zt, int zb, int num_sms, cudaStream_t s);
cudaError_t launch_conv_tb2_r2(const StencilGeom& g, const RowBands& b, int zt, int zb, int num_sms, cudaStream_t s);

bool conv_tb2_supported(int r, int64_t w, int64_t pitch) {
    return (r == 1 || r == 2) && w % 4 == 0 && w >= 4 && pitch % 16 == 0 && !getenv("MAPSM_CONV_NO_TB");
}

cudaError_t launch_conv_tb2(const StencilGeom& g, const RowBands& b, int r, int zero_top, int zero_bot, int num_sms,
                            cudaStream_t s) {
    if (!conv_tb2_supported(r, g.w, g.pitch)) return cudaErrorInvalidValue;
    return r == 1 ? launch_conv_tb2_r1(g, b, zero_top, zero_bot, num_sms, s)
                  : launch_conv_tb2_r2(g, b, zero_top, zero_bot, num_sms, s);
}
cudaError_t conv_upload_weights_r3(int cm, int slot, const float* w);
cudaError_t conv_upload_weights_r4(int cm, int slot, const float* w);

cudaError_t conv_upload_weights(int r, int cm, int slot, const float* w) {
    if (r == 1) return conv_upload_weights_r1(cm, slot, w);
    if (r == 2) return conv_upload_weights_r2(cm, slot, w);
    if (r == 3) return conv_upload_weights_r3(cm, slot, w);
    if (r == 4) return conv_upload_weights_r4(cm, slot, w);
    return cudaSuccess;
}

cudaError_t launch_conv_step(const StencilGeom& g, const RowBands& b, int r, const float* weights, int num_sms,
                             cudaStream_t s, const FusedLink* link) {
    switch (r) {
        case 1: return launch_conv_radius<1>(g, b, weights, num_sms, s, link);
        case 2: return launch_conv_radius<2>(g, b, weights, num_sms, s, link);
        case 3: return launch_conv_radius<3>(g, b, weights, num_sms, s, link);
        case 4: return launch_conv_radius<4>(g, b, weights, num_sms, s, link);
        case 5: case 6: case 7: case 8:
            if (link) return cudaErrorInvalidValue;  // the fused exchange needs the TMA kernels (r <= 4)
            return launch_conv_wide(g, b, r, weights, s);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace mapsm

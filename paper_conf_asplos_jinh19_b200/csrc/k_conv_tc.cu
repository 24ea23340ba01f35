// k_conv_tc.cu -- tcgen05 implicit-GEMM split convolution (placeholder until the kernel lands).
#include "kernels.h"

namespace splitcnn {
bool conv_tc_supported(int, splitcnn_dtype_t, const Level &, const Level &, const LayerGeom &) { return false; }
size_t conv_tc_ws_bytes(int, const Level &, const Level &, const LayerGeom &) { return 0; }
splitcnn_status_t launch_conv_fwd_tc(const Level &, const Level &, const LayerGeom &, const void *, const void *,
                                     const float *, void *, int, int, int, cudaStream_t) { return fail(SPLITCNN_ERR_UNSUPPORTED, "tc"); }
splitcnn_status_t launch_conv_dgrad_tc(const Level &, const Level &, const LayerGeom &, const void *, const void *,
                                       void *, const void *, void *, int, int, cudaStream_t) { return fail(SPLITCNN_ERR_UNSUPPORTED, "tc"); }
splitcnn_status_t launch_conv_wgrad_tc(const Level &, const Level &, const LayerGeom &, const void *, const void *,
                                       float *, float *, float, void *, int, int, cudaStream_t) { return fail(SPLITCNN_ERR_UNSUPPORTED, "tc"); }
}  // namespace splitcnn

// kernels.h -- launchers of the libsplitcnn kernels (library-private).
#pragma once
#include <cuda_runtime.h>

#include "internal.h"

namespace splitcnn {

// k_memops.cu
void launch_split(splitcnn_dtype_t dt, const Level &L, const void *x, int layout, void *P, int p0, int p1, cudaStream_t st,
                  int xc = 0, int row0 = 0, int xH = 0);
void launch_merge(splitcnn_dtype_t dt, const Level &L, const void *P, void *y, int layout, int p0, int p1, cudaStream_t st);
void launch_pool_fwd(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g, const void *x, void *y,
                     uint8_t *a, int relu_bit, int p0, int p1, cudaStream_t st);
void launch_pool_bwd(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g, const void *dy,
                     const uint8_t *a, void *dx, int relu_bit, int p0, int p1, cudaStream_t st);
void launch_gap(splitcnn_dtype_t dt, bool fwd, const Level &L, const void *a, void *b, cudaStream_t st);
void launch_add(splitcnn_dtype_t dt, const void *a, const void *b, void *y, const void *m, int relu, int64_t n,
                cudaStream_t st);

// k_bn.cu
size_t bn_ws_bytes(int C);
void launch_bn_reduce(splitcnn_dtype_t dt, int mode, const void *x, const void *dy, const void *y, const float *mi,
                      int64_t P, int Cpad, int C, float *part, float *sums, cudaStream_t st);
void launch_bn_fwd(splitcnn_dtype_t dt, const void *x, const float *sums, double count, const float *gamma,
                   const float *beta, float eps, float *mi, void *y, int relu, int64_t n, int Cpad, int C,
                   cudaStream_t st);
void launch_bn_bwd(splitcnn_dtype_t dt, const void *dy, const void *x, const void *y, const float *mi,
                   const float *gamma, const float *t, double count, void *dx, int64_t n, int Cpad, int C,
                   cudaStream_t st);

// k_conv_simt.cu
void launch_conv_fwd_simt(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g, const void *x,
                          const void *w, const float *bias, void *y, int relu, int p0, int p1, cudaStream_t st);
void launch_conv_dgrad_simt(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g, const void *dy,
                            const void *w, void *dx, const void *relu_src, int p0, int p1, cudaStream_t st);
void launch_conv_wgrad_simt(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g, const void *x,
                            const void *dy, float *dw, float *db, float beta, void *ws, int p0, int p1, cudaStream_t st);
size_t wgrad_simt_ws_bytes(const Level &Li, const Level &Lo, const LayerGeom &g);

// k_conv_tc.cu (tcgen05); return false when the shape is not supported by the tensor-core path
bool conv_tc_supported(int mode, splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g);
size_t conv_tc_ws_bytes(int mode, const Level &Li, const Level &Lo, const LayerGeom &g, splitcnn_dtype_t dt = SPLITCNN_BF16);
splitcnn_status_t launch_conv_fwd_tc(const Level &Li, const Level &Lo, const LayerGeom &g, const void *x, const void *w,
                                     const float *bias, void *y, int relu, int p0, int p1, cudaStream_t st,
                                     splitcnn_dtype_t dt = SPLITCNN_BF16, int accum = 0);
splitcnn_status_t launch_conv_fwd_res_tc(const Level &Li, const Level &Lo, const LayerGeom &g, const void *x, const void *w,
                                         const float *bias, const void *residual, void *y, int relu, int p0, int p1,
                                         cudaStream_t st);
splitcnn_status_t launch_conv_pool_fwd_tc(const Level &Li, const Level &Lo, const Level &Lp, const LayerGeom &g,
                                          const void *x, const void *w, const float *bias, void *y_pool, uint8_t *argmax,
                                          int p0, int p1, cudaStream_t st);
splitcnn_status_t launch_conv_dgrad_tc(const Level &Li, const Level &Lo, const LayerGeom &g, const void *dy, const void *w,
                                       void *dx, const void *relu_src, void *ws, int p0, int p1, cudaStream_t st,
                                       splitcnn_dtype_t dt = SPLITCNN_BF16, int accum = 0, bool prepared = false);
// the dgrad-ready (flipped / phase) weights launch_conv_dgrad_tc builds in its workspace, into wt (BF16)
// max_blocks <= 0: one block per SM
void prep_dgrad_weights_tc(const Level &Li, const Level &Lo, const LayerGeom &g, const void *w, void *wt, cudaStream_t st,
                           int max_blocks);
splitcnn_status_t launch_conv_wgrad_tc(const Level &Li, const Level &Lo, const LayerGeom &g, const void *x, const void *dy,
                                       float *dw, float *db, float beta, void *ws, int p0, int p1, cudaStream_t st);
// fp32 storage on the tensor cores (TF32 one pass / FP32 3xTF32; wgrad by bf16 operand splitting)
size_t f32tc_ws_bytes(int op, splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g);
splitcnn_status_t launch_conv_fwd_f32tc(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g,
                                        const void *x, const void *w, const float *bias, void *y, int relu, int p0, int p1,
                                        void *ws, cudaStream_t st);
splitcnn_status_t launch_conv_dgrad_f32tc(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g,
                                          const void *dy, const void *w, void *dx, const void *relu_src, int p0, int p1,
                                          void *ws, cudaStream_t st);
splitcnn_status_t launch_conv_wgrad_f32tc(splitcnn_dtype_t dt, const Level &Li, const Level &Lo, const LayerGeom &g,
                                          const void *x, const void *dy, float *dw, float *db, float beta, void *ws,
                                          int p0, int p1, cudaStream_t st);

}  // namespace splitcnn

// api.cu -- the extern "C" entry points of libsplitcnn (see include/splitcnn.h).
// Argument validation, error plumbing and kernel dispatch; all arithmetic is in the kernels.
#include <atomic>
#include <cstdio>
#include <cstring>
#include <string>

#include "kernels.h"

namespace splitcnn {

static thread_local std::string g_last_error;
static std::atomic<uint64_t> g_launches{0};

void count_launch(int n) { g_launches.fetch_add((uint64_t)n, std::memory_order_relaxed); }

void set_error(const std::string &msg) { g_last_error = msg; }

splitcnn_status_t fail(splitcnn_status_t s, const std::string &msg) {
    g_last_error = msg;
    return s;
}

splitcnn_status_t check_launch(const char *what) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return fail(SPLITCNN_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
    return SPLITCNN_OK;
}

}  // namespace splitcnn

using namespace splitcnn;

extern "C" const char *splitcnn_last_error(void) { return g_last_error.c_str(); }

extern "C" const char *splitcnn_status_string(splitcnn_status_t s) {
    switch (s) {
        case SPLITCNN_OK: return "ok";
        case SPLITCNN_ERR_INVALID_VALUE: return "invalid value";
        case SPLITCNN_ERR_ALIGNMENT: return "misaligned pointer";
        case SPLITCNN_ERR_UNSUPPORTED: return "unsupported";
        case SPLITCNN_ERR_CUDA: return "CUDA error";
        case SPLITCNN_ERR_OOM: return "out of memory";
    }
    return "unknown status";
}

extern "C" splitcnn_status_t splitcnn_kernel_launches(uint64_t *count) {
    if (!count) return fail(SPLITCNN_ERR_INVALID_VALUE, "null count");
    *count = g_launches.load(std::memory_order_relaxed);
    return SPLITCNN_OK;
}

extern "C" const char *splitcnn_version(void) { return "splitcnn-b200 0.1 (sm_100a)"; }

namespace {

bool aligned16(const void *p) { return ((uintptr_t)p & 15u) == 0; }

splitcnn_status_t check_dtype(splitcnn_dtype_t dt) {
    if (dt != SPLITCNN_BF16 && dt != SPLITCNN_FP32 && dt != SPLITCNN_TF32) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad dtype");
    return SPLITCNN_OK;
}

splitcnn_status_t check_range(const splitcnn_plan_t plan, int level, int &p0, int &p1) {
    const Level &L = plan->levels[level];
    if (p1 < 0) p1 = L.npatch();
    if (p0 < 0 || p0 > p1 || p1 > L.npatch()) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad patch range");
    return SPLITCNN_OK;
}

splitcnn_status_t check_layer(const splitcnn_plan_t plan, int layer, int op) {
    if (!plan) return fail(SPLITCNN_ERR_INVALID_VALUE, "null plan");
    if (layer < 0 || layer >= (int)plan->layers.size()) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad layer index");
    if (plan->layers[layer].L.op != op)
        return fail(SPLITCNN_ERR_INVALID_VALUE, op == SPLITCNN_OP_CONV ? "layer is not a convolution" : "layer is not a max-pool");
    return SPLITCNN_OK;
}

#define TRY(x)                                  \
    do {                                        \
        splitcnn_status_t _s = (x);             \
        if (_s != SPLITCNN_OK) return _s;       \
    } while (0)

#define NEED_ALIGNED(p, name)                                                              \
    do {                                                                                   \
        if ((p) && !aligned16(p)) return fail(SPLITCNN_ERR_ALIGNMENT, name " must be 16-byte aligned"); \
    } while (0)

}  // namespace

extern "C" splitcnn_status_t splitcnn_workspace_size(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                                     int32_t op, size_t *bytes) {
    if (!bytes) return fail(SPLITCNN_ERR_INVALID_VALUE, "null bytes");
    TRY(check_dtype(dtype));
    TRY(check_layer(plan, layer, SPLITCNN_OP_CONV));
    const Level &Li = plan->levels[layer], &Lo = plan->levels[layer + 1];
    const LayerGeom &g = plan->layers[layer];
    size_t b = 0;
    const bool f32 = dtype != SPLITCNN_BF16;
    if (op == 0) {
        if (f32 && conv_tc_supported(0, dtype, Li, Lo, g)) b = f32tc_ws_bytes(0, dtype, Li, Lo, g);
    } else if (op == 1) {
        if (conv_tc_supported(1, dtype, Li, Lo, g)) b = f32 ? f32tc_ws_bytes(1, dtype, Li, Lo, g) : conv_tc_ws_bytes(1, Li, Lo, g);
    } else if (op == 2) {
        b = wgrad_simt_ws_bytes(Li, Lo, g);
        if (conv_tc_supported(2, SPLITCNN_BF16, Li, Lo, g))
            b = std::max(b, f32 ? f32tc_ws_bytes(2, dtype, Li, Lo, g) : conv_tc_ws_bytes(2, Li, Lo, g));
    } else {
        return fail(SPLITCNN_ERR_INVALID_VALUE, "workspace_size: op must be 0, 1 or 2");
    }
    *bytes = b;
    return SPLITCNN_OK;
}

extern "C" splitcnn_status_t splitcnn_split(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype, const void *x,
                                            int32_t x_layout, void *patches, int32_t p0, int32_t p1,
                                            splitcnn_stream_t stream) {
    if (!plan || level < 0 || level >= (int)plan->levels.size()) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad level");
    TRY(check_dtype(dtype));
    if (!x || !patches) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    if (x_layout != SPLITCNN_NCHW && x_layout != SPLITCNN_NHWC && x_layout != SPLITCNN_NCHW_S2D)
        return fail(SPLITCNN_ERR_INVALID_VALUE, "bad layout");
    if (x_layout == SPLITCNN_NCHW_S2D && plan->levels[level].C % 4)
        return fail(SPLITCNN_ERR_INVALID_VALUE, "space-to-depth split needs C % 4 == 0");
    NEED_ALIGNED(x, "x");
    NEED_ALIGNED(patches, "patches");
    TRY(check_range(plan, level, p0, p1));
    if (p1 == p0) return SPLITCNN_OK;
    launch_split(dtype, plan->levels[level], x, x_layout, patches, p0, p1, (cudaStream_t)stream);
    return check_launch("split");
}

extern "C" splitcnn_status_t splitcnn_split_rows(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                                 const void *x, int32_t x_layout, int32_t row0, int32_t row1,
                                                 void *patches, int32_t p0, int32_t p1, splitcnn_stream_t stream) {
    if (!plan || level < 0 || level >= (int)plan->levels.size()) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad level");
    TRY(check_dtype(dtype));
    if (!x || !patches) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    if (x_layout != SPLITCNN_NCHW && x_layout != SPLITCNN_NHWC)
        return fail(SPLITCNN_ERR_INVALID_VALUE, "split_rows: layout must be NCHW or NHWC");
    NEED_ALIGNED(x, "x");
    NEED_ALIGNED(patches, "patches");
    TRY(check_range(plan, level, p0, p1));
    const Level &L = plan->levels[level];
    if (row0 < 0 || row1 > L.H || row0 >= row1) return fail(SPLITCNN_ERR_INVALID_VALUE, "split_rows: bad row window");
    if (p1 == p0) return SPLITCNN_OK;
    const int i0 = p0 / L.nw(), i1 = (p1 - 1) / L.nw();
    if (L.bh[i0] < row0 || L.bh[i1 + 1] > row1)
        return fail(SPLITCNN_ERR_INVALID_VALUE, "split_rows: a patch of [p0, p1) reads rows outside [row0, row1)");
    launch_split(dtype, L, x, x_layout, patches, p0, p1, (cudaStream_t)stream, 0, row0, row1 - row0);
    return check_launch("split_rows");
}

extern "C" splitcnn_status_t splitcnn_split_s2d(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                                const void *x, int32_t x_channels, void *patches, int32_t p0,
                                                int32_t p1, splitcnn_stream_t stream) {
    if (!plan || level < 0 || level >= (int)plan->levels.size()) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad level");
    TRY(check_dtype(dtype));
    if (!x || !patches) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    if (x_channels < 1 || 4 * x_channels > plan->levels[level].C)
        return fail(SPLITCNN_ERR_INVALID_VALUE, "split_s2d: need 1 <= x_channels and 4 * x_channels <= level C");
    NEED_ALIGNED(x, "x");
    NEED_ALIGNED(patches, "patches");
    TRY(check_range(plan, level, p0, p1));
    if (p1 == p0) return SPLITCNN_OK;
    launch_split(dtype, plan->levels[level], x, SPLITCNN_NCHW_S2D, patches, p0, p1, (cudaStream_t)stream, x_channels);
    return check_launch("split_s2d");
}

extern "C" splitcnn_status_t splitcnn_merge(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                            const void *patches, void *y, int32_t y_layout, int32_t p0, int32_t p1,
                                            splitcnn_stream_t stream) {
    if (!plan || level < 0 || level >= (int)plan->levels.size()) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad level");
    TRY(check_dtype(dtype));
    if (!y || !patches) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    if (y_layout != SPLITCNN_NCHW && y_layout != SPLITCNN_NHWC) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad layout");
    NEED_ALIGNED(y, "y");
    NEED_ALIGNED(patches, "patches");
    TRY(check_range(plan, level, p0, p1));
    if (p1 == p0) return SPLITCNN_OK;
    launch_merge(dtype, plan->levels[level], patches, y, y_layout, p0, p1, (cudaStream_t)stream);
    return check_launch("merge");
}

extern "C" splitcnn_status_t splitcnn_conv_fwd_ws(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                                  const void *x, const void *w, const float *bias, void *y,
                                                  uint32_t flags, void *ws, size_t ws_bytes, int32_t p0, int32_t p1,
                                                  splitcnn_stream_t stream) {
    TRY(check_layer(plan, layer, SPLITCNN_OP_CONV));
    TRY(check_dtype(dtype));
    if (!x || !w || !y) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    NEED_ALIGNED(x, "x");
    NEED_ALIGNED(w, "w");
    NEED_ALIGNED(y, "y");
    NEED_ALIGNED(ws, "ws");
    TRY(check_range(plan, layer, p0, p1));
    if (p1 == p0) return SPLITCNN_OK;
    const Level &Li = plan->levels[layer], &Lo = plan->levels[layer + 1];
    const LayerGeom &g = plan->layers[layer];
    const int relu = (flags & SPLITCNN_FLAG_RELU) ? 1 : 0;
    const bool tc = !(flags & SPLITCNN_FLAG_FORCE_SIMT) && conv_tc_supported(0, dtype, Li, Lo, g);
    if (tc && dtype == SPLITCNN_BF16) {
        TRY(launch_conv_fwd_tc(Li, Lo, g, x, w, bias, y, relu, p0, p1, (cudaStream_t)stream));
    } else if (tc && (dtype == SPLITCNN_TF32 || (ws && ws_bytes >= f32tc_ws_bytes(0, dtype, Li, Lo, g)))) {
        // TF32: one kind::tf32 pass; FP32 with a workspace: 3xTF32 (without one: FFMA below)
        TRY(launch_conv_fwd_f32tc(dtype, Li, Lo, g, x, w, bias, y, relu, p0, p1, ws, (cudaStream_t)stream));
    } else {
        launch_conv_fwd_simt(dtype, Li, Lo, g, x, w, bias, y, relu, p0, p1, (cudaStream_t)stream);
    }
    return check_launch("conv_fwd");
}

extern "C" splitcnn_status_t splitcnn_conv_fwd_res(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                                   const void *x, const void *w, const float *bias, const void *residual,
                                                   void *y, uint32_t flags, void *ws, size_t ws_bytes, int32_t p0,
                                                   int32_t p1, splitcnn_stream_t stream) {
    TRY(check_layer(plan, layer, SPLITCNN_OP_CONV));
    TRY(check_dtype(dtype));
    if (!x || !w || !y || !residual) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    if (residual == y) return fail(SPLITCNN_ERR_INVALID_VALUE, "conv_fwd_res: residual must not alias y");
    NEED_ALIGNED(residual, "residual");
    TRY(check_range(plan, layer, p0, p1));
    if (p1 == p0) return SPLITCNN_OK;
    const Level &Li = plan->levels[layer], &Lo = plan->levels[layer + 1];
    const LayerGeom &g = plan->layers[layer];
    const int relu = (flags & SPLITCNN_FLAG_RELU) ? 1 : 0;
    if (dtype == SPLITCNN_BF16 && !(flags & SPLITCNN_FLAG_FORCE_SIMT) && conv_tc_supported(0, dtype, Li, Lo, g)) {
        const splitcnn_status_t r = launch_conv_fwd_res_tc(Li, Lo, g, x, w, bias, residual, y, relu, p0, p1,
                                                           (cudaStream_t)stream);
        if (r == SPLITCNN_OK) return check_launch("conv_fwd_res");
        if (r != SPLITCNN_ERR_UNSUPPORTED) return r;
    }
    // other shapes / precisions: the conv (no activation) into y, then y = act(y + residual)
    TRY(splitcnn_conv_fwd_ws(plan, layer, dtype, x, w, bias, y, flags & ~SPLITCNN_FLAG_RELU, ws, ws_bytes, p0, p1,
                             stream));
    return splitcnn_add(plan, layer + 1, dtype, y, residual, y, nullptr, relu ? SPLITCNN_FLAG_RELU : 0u, p0, p1, stream);
}

extern "C" splitcnn_status_t splitcnn_conv_fwd(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype, const void *x,
                                               const void *w, const float *bias, void *y, uint32_t flags, int32_t p0,
                                               int32_t p1, splitcnn_stream_t stream) {
    return splitcnn_conv_fwd_ws(plan, layer, dtype, x, w, bias, y, flags, nullptr, 0, p0, p1, stream);
}

// conv `layer` (+bias, ReLU) followed by a 2x2 / stride-2 / unpadded max-pool `layer + 1` whose
// epilogue the tcgen05 kernel can take
static bool conv_pool_fusable(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype) {
    if (layer < 0 || layer + 1 >= (int)plan->layers.size()) return false;
    const LayerGeom &g = plan->layers[layer], &q = plan->layers[layer + 1];
    if (g.L.op != SPLITCNN_OP_CONV || q.L.op != SPLITCNN_OP_MAXPOOL) return false;
    if (q.L.kh != 2 || q.L.kw != 2 || q.L.sh != 2 || q.L.sw != 2) return false;
    for (int v : q.pad_h) if (v) return false;
    for (int v : q.pad_w) if (v) return false;
    const Level &Li = plan->levels[layer], &Lo = plan->levels[layer + 1];
    if (!conv_tc_supported(0, dtype, Li, Lo, g)) return false;
    if (Li.Cpad == 8 && g.L.sh == 1) return false;            // 8-channel halo path: no fused variant
    if (g.L.cout != Lo.Cpad || g.L.cout % 16) return false;   // every stored channel is a real one
    return true;
}

extern "C" splitcnn_status_t splitcnn_conv_pool_supported(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                                          int32_t *supported) {
    if (!plan || !supported) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    TRY(check_dtype(dtype));
    *supported = conv_pool_fusable(plan, layer, dtype) ? 1 : 0;
    return SPLITCNN_OK;
}

extern "C" splitcnn_status_t splitcnn_conv_pool_fwd(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                                    const void *x, const void *w, const float *bias, void *y_pool,
                                                    uint8_t *argmax, uint32_t flags, int32_t p0, int32_t p1,
                                                    splitcnn_stream_t stream) {
    TRY(check_layer(plan, layer, SPLITCNN_OP_CONV));
    TRY(check_dtype(dtype));
    if (!x || !w || !y_pool || !argmax) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    NEED_ALIGNED(x, "x");
    NEED_ALIGNED(w, "w");
    NEED_ALIGNED(y_pool, "y_pool");
    NEED_ALIGNED(argmax, "argmax");
    const uint32_t need = SPLITCNN_FLAG_RELU | SPLITCNN_FLAG_POOL_RELU_MASK;
    if ((flags & need) != need || (flags & SPLITCNN_FLAG_FORCE_SIMT) || !conv_pool_fusable(plan, layer, dtype))
        return fail(SPLITCNN_ERR_UNSUPPORTED, "conv_pool_fwd: not a fusable conv(+ReLU) -> 2x2/s2 max-pool pair");
    TRY(check_range(plan, layer, p0, p1));
    if (p1 == p0) return SPLITCNN_OK;
    TRY(launch_conv_pool_fwd_tc(plan->levels[layer], plan->levels[layer + 1], plan->levels[layer + 2], plan->layers[layer],
                                x, w, bias, y_pool, argmax, p0, p1, (cudaStream_t)stream));
    return check_launch("conv_pool_fwd");
}

extern "C" splitcnn_status_t splitcnn_conv_bwd_data(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                                    const void *dy, const void *w, void *dx, const void *relu_src,
                                                    void *ws, size_t ws_bytes, uint32_t flags, int32_t p0, int32_t p1,
                                                    splitcnn_stream_t stream) {
    TRY(check_layer(plan, layer, SPLITCNN_OP_CONV));
    TRY(check_dtype(dtype));
    if (!dy || !w || !dx) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    NEED_ALIGNED(dy, "dy");
    NEED_ALIGNED(w, "w");
    NEED_ALIGNED(dx, "dx");
    NEED_ALIGNED(relu_src, "relu_src");
    NEED_ALIGNED(ws, "ws");
    TRY(check_range(plan, layer, p0, p1));
    if (p1 == p0) return SPLITCNN_OK;
    const Level &Li = plan->levels[layer], &Lo = plan->levels[layer + 1];
    const LayerGeom &g = plan->layers[layer];
    const bool prepared = (flags & SPLITCNN_FLAG_DGRAD_WEIGHTS) != 0;
    const bool tc = !(flags & SPLITCNN_FLAG_FORCE_SIMT) && conv_tc_supported(1, dtype, Li, Lo, g);
    if (prepared && !(tc && dtype == SPLITCNN_BF16))
        return fail(SPLITCNN_ERR_INVALID_VALUE, "conv_bwd_data: FLAG_DGRAD_WEIGHTS where the data gradient takes none "
                                                "(splitcnn_conv_dgrad_weights_size = 0)");
    if (prepared) {   // w = splitcnn_conv_dgrad_weights output: no flip, no workspace
        TRY(launch_conv_dgrad_tc(Li, Lo, g, dy, w, dx, relu_src, nullptr, p0, p1, (cudaStream_t)stream, SPLITCNN_BF16, 0, true));
    } else if (tc) {
        const bool f32 = dtype != SPLITCNN_BF16;
        const size_t need = f32 ? f32tc_ws_bytes(1, dtype, Li, Lo, g) : conv_tc_ws_bytes(1, Li, Lo, g);
        if (ws_bytes < need || (need && !ws)) return fail(SPLITCNN_ERR_INVALID_VALUE, "conv_bwd_data: workspace too small");
        if (f32) TRY(launch_conv_dgrad_f32tc(dtype, Li, Lo, g, dy, w, dx, relu_src, p0, p1, ws, (cudaStream_t)stream));
        else TRY(launch_conv_dgrad_tc(Li, Lo, g, dy, w, dx, relu_src, ws, p0, p1, (cudaStream_t)stream));
    } else {
        launch_conv_dgrad_simt(dtype, Li, Lo, g, dy, w, dx, relu_src, p0, p1, (cudaStream_t)stream);
    }
    return check_launch("conv_bwd_data");
}

extern "C" splitcnn_status_t splitcnn_conv_dgrad_weights_size(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                                             size_t *bytes) {
    TRY(check_layer(plan, layer, SPLITCNN_OP_CONV));
    TRY(check_dtype(dtype));
    if (!bytes) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    const Level &Li = plan->levels[layer], &Lo = plan->levels[layer + 1];
    const LayerGeom &g = plan->layers[layer];
    *bytes = (dtype == SPLITCNN_BF16 && conv_tc_supported(1, dtype, Li, Lo, g)) ? conv_tc_ws_bytes(1, Li, Lo, g) : 0;
    return SPLITCNN_OK;
}

extern "C" splitcnn_status_t splitcnn_conv_dgrad_weights(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                                        const void *w, void *wt, size_t wt_bytes, splitcnn_stream_t stream) {
    size_t need = 0;
    TRY(splitcnn_conv_dgrad_weights_size(plan, layer, dtype, &need));
    if (need == 0) return fail(SPLITCNN_ERR_UNSUPPORTED, "conv_dgrad_weights: this layer / dtype takes no prepared weights");
    if (!w || !wt) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    NEED_ALIGNED(w, "w");
    NEED_ALIGNED(wt, "wt");
    if (wt_bytes < need) return fail(SPLITCNN_ERR_INVALID_VALUE, "conv_dgrad_weights: wt too small");
    prep_dgrad_weights_tc(plan->levels[layer], plan->levels[layer + 1], plan->layers[layer], w, wt, (cudaStream_t)stream, 0);
    return check_launch("conv_dgrad_weights");
}

extern "C" splitcnn_status_t splitcnn_conv_bwd_filter(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                                      const void *x, const void *dy, float *dw, float *db, float beta,
                                                      void *ws, size_t ws_bytes, uint32_t flags, int32_t p0, int32_t p1,
                                                      splitcnn_stream_t stream) {
    TRY(check_layer(plan, layer, SPLITCNN_OP_CONV));
    TRY(check_dtype(dtype));
    if (!x || !dy || !dw) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    if (beta != 0.f && beta != 1.f) return fail(SPLITCNN_ERR_INVALID_VALUE, "beta must be 0 or 1");
    NEED_ALIGNED(x, "x");
    NEED_ALIGNED(dy, "dy");
    NEED_ALIGNED(dw, "dw");
    NEED_ALIGNED(ws, "ws");
    TRY(check_range(plan, layer, p0, p1));
    const Level &Li = plan->levels[layer], &Lo = plan->levels[layer + 1];
    const LayerGeom &g = plan->layers[layer];
    // fp32 storage: bf16 operand splitting onto the bf16 tensor-core kernels where they take the shape
    const bool f32 = dtype != SPLITCNN_BF16;
    const bool tc = !(flags & SPLITCNN_FLAG_FORCE_SIMT) && conv_tc_supported(2, SPLITCNN_BF16, Li, Lo, g);
    const size_t need = !tc ? wgrad_simt_ws_bytes(Li, Lo, g) : f32 ? f32tc_ws_bytes(2, dtype, Li, Lo, g)
                                                                   : conv_tc_ws_bytes(2, Li, Lo, g);
    if (ws_bytes < need || !ws) return fail(SPLITCNN_ERR_INVALID_VALUE, "conv_bwd_filter: workspace too small");
    if (tc && f32) {
        TRY(launch_conv_wgrad_f32tc(dtype, Li, Lo, g, x, dy, dw, db, beta, ws, p0, p1, (cudaStream_t)stream));
    } else if (tc) {
        TRY(launch_conv_wgrad_tc(Li, Lo, g, x, dy, dw, db, beta, ws, p0, p1, (cudaStream_t)stream));
    } else {
        launch_conv_wgrad_simt(dtype, Li, Lo, g, x, dy, dw, db, beta, ws, p0, p1, (cudaStream_t)stream);
    }
    return check_launch("conv_bwd_filter");
}

extern "C" splitcnn_status_t splitcnn_pool_fwd(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype, const void *x,
                                               void *y, uint8_t *argmax, uint32_t flags, int32_t p0, int32_t p1,
                                               splitcnn_stream_t stream) {
    TRY(check_layer(plan, layer, SPLITCNN_OP_MAXPOOL));
    TRY(check_dtype(dtype));
    if (!x || !y || !argmax) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    NEED_ALIGNED(x, "x");
    NEED_ALIGNED(y, "y");
    NEED_ALIGNED(argmax, "argmax");
    TRY(check_range(plan, layer, p0, p1));
    if (p1 == p0) return SPLITCNN_OK;
    launch_pool_fwd(dtype, plan->levels[layer], plan->levels[layer + 1], plan->layers[layer], x, y, argmax,
                    (flags & SPLITCNN_FLAG_POOL_RELU_MASK) ? 1 : 0, p0, p1, (cudaStream_t)stream);
    return check_launch("pool_fwd");
}

extern "C" splitcnn_status_t splitcnn_pool_bwd(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype, const void *dy,
                                               const uint8_t *argmax, void *dx, uint32_t flags, int32_t p0, int32_t p1,
                                               splitcnn_stream_t stream) {
    TRY(check_layer(plan, layer, SPLITCNN_OP_MAXPOOL));
    TRY(check_dtype(dtype));
    if (!dy || !dx || !argmax) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    NEED_ALIGNED(dy, "dy");
    NEED_ALIGNED(dx, "dx");
    NEED_ALIGNED(argmax, "argmax");
    TRY(check_range(plan, layer, p0, p1));
    if (p1 == p0) return SPLITCNN_OK;
    launch_pool_bwd(dtype, plan->levels[layer], plan->levels[layer + 1], plan->layers[layer], dy, argmax, dx,
                    (flags & SPLITCNN_FLAG_POOL_RELU_MASK) ? 1 : 0, p0, p1, (cudaStream_t)stream);
    return check_launch("pool_bwd");
}

// ------------------------------------------------------------------ residual add
extern "C" splitcnn_status_t splitcnn_add(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype, const void *a,
                                          const void *b, void *y, const void *mask, uint32_t flags, int32_t p0,
                                          int32_t p1, splitcnn_stream_t stream) {
    if (!plan || level < 0 || level >= (int)plan->levels.size()) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad level");
    TRY(check_dtype(dtype));
    if (!a || !y || (!b && !mask)) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    if (mask && (flags & SPLITCNN_FLAG_RELU)) return fail(SPLITCNN_ERR_INVALID_VALUE, "FLAG_RELU with a mask");
    NEED_ALIGNED(a, "a");
    NEED_ALIGNED(b, "b");
    NEED_ALIGNED(y, "y");
    NEED_ALIGNED(mask, "mask");
    TRY(check_range(plan, level, p0, p1));
    if (p1 == p0) return SPLITCNN_OK;
    const Level &L = plan->levels[level];
    auto off = [&](int p) { return p == L.npatch() ? L.total() : L.offset(p / L.nw(), p % L.nw()); };
    const int64_t o0 = off(p0), n = off(p1) - o0;
    const size_t es = dtype == SPLITCNN_BF16 ? 2 : 4;
    auto at = [&](const void *p) { return p ? (const void *)((const char *)p + o0 * es) : nullptr; };
    launch_add(dtype, at(a), at(b), (void *)at(y), at(mask), (flags & SPLITCNN_FLAG_RELU) ? 1 : 0, n,
               (cudaStream_t)stream);
    return check_launch("add");
}

// ------------------------------------------------------------------ global average pool
extern "C" splitcnn_status_t splitcnn_gap_fwd(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                              const void *x, void *y, splitcnn_stream_t stream) {
    if (!plan || level < 0 || level >= (int)plan->levels.size()) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad level");
    TRY(check_dtype(dtype));
    if (!x || !y) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    NEED_ALIGNED(x, "x");
    NEED_ALIGNED(y, "y");
    launch_gap(dtype, true, plan->levels[level], x, y, (cudaStream_t)stream);
    return check_launch("gap_fwd");
}

extern "C" splitcnn_status_t splitcnn_gap_bwd(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                              const void *dy, void *dx, splitcnn_stream_t stream) {
    if (!plan || level < 0 || level >= (int)plan->levels.size()) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad level");
    TRY(check_dtype(dtype));
    if (!dy || !dx) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    NEED_ALIGNED(dy, "dy");
    NEED_ALIGNED(dx, "dx");
    launch_gap(dtype, false, plan->levels[level], dy, dx, (cudaStream_t)stream);
    return check_launch("gap_bwd");
}

// ------------------------------------------------------------------ batch normalisation
namespace {
splitcnn_status_t bn_span(splitcnn_plan_t plan, int level, splitcnn_dtype_t dtype, int &p0, int &p1, int64_t &o0,
                          int64_t &n) {
    if (!plan || level < 0 || level >= (int)plan->levels.size()) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad level");
    TRY(check_dtype(dtype));
    TRY(check_range(plan, level, p0, p1));
    const Level &L = plan->levels[level];
    if (L.Cpad > 2048) return fail(SPLITCNN_ERR_UNSUPPORTED, "bn: Cpad > 2048");
    auto off = [&](int p) { return p == L.npatch() ? L.total() : L.offset(p / L.nw(), p % L.nw()); };
    o0 = off(p0);
    n = off(p1) - o0;
    return SPLITCNN_OK;
}
const void *at_(const void *p, int64_t o, splitcnn_dtype_t dt) {
    return p ? (const void *)((const char *)p + o * (dt == SPLITCNN_BF16 ? 2 : 4)) : nullptr;
}
}  // namespace

extern "C" splitcnn_status_t splitcnn_bn_workspace_size(splitcnn_plan_t plan, int32_t level, size_t *bytes) {
    if (!plan || level < 0 || level >= (int)plan->levels.size() || !bytes)
        return fail(SPLITCNN_ERR_INVALID_VALUE, "bad argument");
    *bytes = bn_ws_bytes(plan->levels[level].C);
    return SPLITCNN_OK;
}

extern "C" splitcnn_status_t splitcnn_bn_stats(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                               const void *x, float *sums, void *ws, size_t ws_bytes, int32_t p0,
                                               int32_t p1, splitcnn_stream_t stream) {
    int64_t o0, n;
    TRY(bn_span(plan, level, dtype, p0, p1, o0, n));
    if (!x || !sums || !ws) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    NEED_ALIGNED(x, "x");
    const Level &L = plan->levels[level];
    if (ws_bytes < bn_ws_bytes(L.C)) return fail(SPLITCNN_ERR_INVALID_VALUE, "bn_stats: workspace too small");
    if (n == 0) return cudaMemsetAsync(sums, 0, 2 * L.C * sizeof(float), (cudaStream_t)stream) == cudaSuccess
                           ? SPLITCNN_OK : fail(SPLITCNN_ERR_CUDA, "memset");
    launch_bn_reduce(dtype, 0, at_(x, o0, dtype), nullptr, nullptr, nullptr, n / L.Cpad, L.Cpad, L.C, (float *)ws, sums,
                     (cudaStream_t)stream);
    return check_launch("bn_stats");
}

extern "C" splitcnn_status_t splitcnn_bn_fwd(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                             const void *x, const float *sums, double count, const float *gamma,
                                             const float *beta, float eps, float *mean_invstd, void *y,
                                             uint32_t flags, int32_t p0, int32_t p1, splitcnn_stream_t stream) {
    int64_t o0, n;
    TRY(bn_span(plan, level, dtype, p0, p1, o0, n));
    if (!x || !sums || !gamma || !beta || !mean_invstd || !y) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    if (!(count > 0)) return fail(SPLITCNN_ERR_INVALID_VALUE, "bn_fwd: count must be > 0");
    NEED_ALIGNED(x, "x");
    NEED_ALIGNED(y, "y");
    const Level &L = plan->levels[level];
    launch_bn_fwd(dtype, at_(x, o0, dtype), sums, count, gamma, beta, eps, mean_invstd, (void *)at_(y, o0, dtype),
                  (flags & SPLITCNN_FLAG_RELU) ? 1 : 0, n, L.Cpad, L.C, (cudaStream_t)stream);
    return check_launch("bn_fwd");
}

extern "C" splitcnn_status_t splitcnn_bn_bwd_sums(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                                  const void *dy, const void *x, const void *y,
                                                  const float *mean_invstd, float *t, void *ws, size_t ws_bytes,
                                                  int32_t p0, int32_t p1, splitcnn_stream_t stream) {
    int64_t o0, n;
    TRY(bn_span(plan, level, dtype, p0, p1, o0, n));
    if (!dy || !x || !mean_invstd || !t || !ws) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    NEED_ALIGNED(dy, "dy");
    NEED_ALIGNED(x, "x");
    NEED_ALIGNED(y, "y");
    const Level &L = plan->levels[level];
    if (ws_bytes < bn_ws_bytes(L.C)) return fail(SPLITCNN_ERR_INVALID_VALUE, "bn_bwd_sums: workspace too small");
    if (n == 0) return cudaMemsetAsync(t, 0, 2 * L.C * sizeof(float), (cudaStream_t)stream) == cudaSuccess
                           ? SPLITCNN_OK : fail(SPLITCNN_ERR_CUDA, "memset");
    launch_bn_reduce(dtype, 1, at_(x, o0, dtype), at_(dy, o0, dtype), at_(y, o0, dtype), mean_invstd, n / L.Cpad,
                     L.Cpad, L.C, (float *)ws, t, (cudaStream_t)stream);
    return check_launch("bn_bwd_sums");
}

extern "C" splitcnn_status_t splitcnn_bn_bwd(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                             const void *dy, const void *x, const void *y, const float *mean_invstd,
                                             const float *gamma, const float *t, double count, void *dx, int32_t p0,
                                             int32_t p1, splitcnn_stream_t stream) {
    int64_t o0, n;
    TRY(bn_span(plan, level, dtype, p0, p1, o0, n));
    if (!dy || !x || !mean_invstd || !gamma || !t || !dx) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    if (!(count > 0)) return fail(SPLITCNN_ERR_INVALID_VALUE, "bn_bwd: count must be > 0");
    NEED_ALIGNED(dy, "dy");
    NEED_ALIGNED(x, "x");
    NEED_ALIGNED(y, "y");
    NEED_ALIGNED(dx, "dx");
    if (n == 0) return SPLITCNN_OK;
    const Level &L = plan->levels[level];
    launch_bn_bwd(dtype, at_(dy, o0, dtype), at_(x, o0, dtype), at_(y, o0, dtype), mean_invstd, gamma, t, count,
                  (void *)at_(dx, o0, dtype), n, L.Cpad, L.C, (cudaStream_t)stream);
    return check_launch("bn_bwd");
}

// ------------------------------------------------------------------ offload / prefetch
extern "C" splitcnn_status_t splitcnn_patch_bytes(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                                  int32_t patch, size_t *offset, size_t *bytes) {
    if (!plan || level < 0 || level >= (int)plan->levels.size()) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad level");
    TRY(check_dtype(dtype));
    const Level &L = plan->levels[level];
    if (patch < 0 || patch >= L.npatch()) return fail(SPLITCNN_ERR_INVALID_VALUE, "bad patch");
    const size_t es = dtype == SPLITCNN_BF16 ? 2 : 4;
    const int i = patch / L.nw(), j = patch % L.nw();
    if (offset) *offset = (size_t)L.offset(i, j) * es;
    if (bytes) *bytes = (size_t)L.patch_elems(i, j) * es;
    return SPLITCNN_OK;
}

static splitcnn_status_t copy_patch(splitcnn_plan_t plan, int level, splitcnn_dtype_t dtype, int patch, const void *src,
                                    void *dst, bool d2h, splitcnn_event_t ready, splitcnn_stream_t st,
                                    splitcnn_event_t done) {
    size_t off = 0, bytes = 0;
    TRY(splitcnn_patch_bytes(plan, level, dtype, patch, &off, &bytes));
    if (!src || !dst) return fail(SPLITCNN_ERR_INVALID_VALUE, "null pointer");
    const void *host = d2h ? dst : src;
    cudaPointerAttributes attr;
    if (cudaPointerGetAttributes(&attr, host) != cudaSuccess || attr.type != cudaMemoryTypeHost) {
        cudaGetLastError();
        return fail(SPLITCNN_ERR_INVALID_VALUE, "host buffer is not page-locked (pinned)");
    }
    cudaStream_t s = (cudaStream_t)st;
    if (ready && cudaStreamWaitEvent(s, (cudaEvent_t)ready, 0) != cudaSuccess) return check_launch("offload: wait");
    cudaError_t e;
    if (d2h) e = cudaMemcpyAsync(dst, (const char *)src + off, bytes, cudaMemcpyDeviceToHost, s);
    else e = cudaMemcpyAsync((char *)dst + off, src, bytes, cudaMemcpyHostToDevice, s);
    if (e != cudaSuccess) return fail(SPLITCNN_ERR_CUDA, std::string("offload copy: ") + cudaGetErrorString(e));
    if (done && cudaEventRecord((cudaEvent_t)done, s) != cudaSuccess) return check_launch("offload: record");
    return SPLITCNN_OK;
}

extern "C" splitcnn_status_t splitcnn_offload(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype, int32_t patch,
                                              const void *dev_patches, void *host_pinned, splitcnn_event_t ready,
                                              splitcnn_stream_t mem_stream, splitcnn_event_t done) {
    return copy_patch(plan, level, dtype, patch, dev_patches, host_pinned, true, ready, mem_stream, done);
}

extern "C" splitcnn_status_t splitcnn_prefetch(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype, int32_t patch,
                                               const void *host_pinned, void *dev_patches, splitcnn_event_t ready,
                                               splitcnn_stream_t mem_stream, splitcnn_event_t done) {
    return copy_patch(plan, level, dtype, patch, host_pinned, dev_patches, false, ready, mem_stream, done);
}

// ------------------------------------------------------------------ Algorithm 1 + reverse
extern "C" splitcnn_status_t splitcnn_offload_plan(int32_t T, const double *op_time_s, const int64_t *cand_bytes,
                                                   double bw, int32_t *offload, int32_t *sync_at) {
    if (T < 1 || !op_time_s || !cand_bytes || !offload || !sync_at || !(bw > 0))
        return fail(SPLITCNN_ERR_INVALID_VALUE, "offload_plan: bad argument");
    double cap = 0;  // theoretical limit: sum of t_op * BW
    for (int t = 0; t < T; ++t) cap += op_time_s[t] * bw;
    double balance = 0, offloaded = 0;
    int pending = 0;
    for (int t = 0; t < T; ++t) {
        offload[t] = 0;
        sync_at[t] = 0;
        if (cand_bytes[t] > 0 && offloaded + (double)cand_bytes[t] <= cap) {  // ratio cap (R15)
            offload[t] = 1;
            ++pending;
            balance -= (double)cand_bytes[t];  // loss = TSO size
            offloaded += (double)cand_bytes[t];
        }
        balance += op_time_s[t] * bw;  // gain = t_op * BW
        if (balance >= 0 || t == T - 1) {
            if (pending) sync_at[t] = 1;  // end of offload for every TSO in TSO_to_free
            pending = 0;
            balance = 0;  // R15: no outstanding copy -> no carried capacity
        }
    }
    return SPLITCNN_OK;
}

extern "C" splitcnn_status_t splitcnn_prefetch_plan(int32_t T, const double *op_time_s, const int64_t *need_bytes,
                                                    double bw, int32_t *prefetch_start) {
    if (T < 1 || !op_time_s || !need_bytes || !prefetch_start || !(bw > 0))
        return fail(SPLITCNN_ERR_INVALID_VALUE, "prefetch_plan: bad argument");
    double balance = 0;
    std::vector<int> pend;
    for (int t = 0; t < T; ++t) prefetch_start[t] = -1;
    for (int t = T - 1; t >= 0; --t) {
        if (!pend.empty()) {
            balance += op_time_s[t] * bw;  // op t runs while the prefetch is in flight
            if (balance >= 0) {
                for (int u : pend) prefetch_start[u] = t;
                pend.clear();
                balance = 0;
            }
        }
        if (need_bytes[t] > 0) {
            pend.push_back(t);
            balance -= (double)need_bytes[t];
        }
    }
    for (int u : pend) prefetch_start[u] = 0;  // cannot be hidden: start at the first backward op
    return SPLITCNN_OK;
}

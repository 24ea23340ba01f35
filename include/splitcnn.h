/*
 * splitcnn.h -- C ABI of the B200-native Split-CNN split window-operator library
 * (libsplitcnn.so, sm_100a).
 *
 * Split-CNN (Jin & Hong, ASPLOS'19; /root/reference/PAPER.md, cited P:<line>)
 * cuts the input of early CNN layers into spatial patches and runs every
 * window operator (convolution, max-pool) on each patch independently with
 * patch-local padding, so no window crosses a patch boundary:
 *
 *   I = ComputeInputSplitScheme(k, s, p, O)        Eq. 3, Eq. 1-2
 *   X_0..X_{N-1} = Split_W(X, I)                   Eq. 4
 *   p = ComputePadding(k, s, p, O, I)              Eq. 5
 *   Y_n = Op(X_n, k, s, p_n)                       Eq. 6
 *   Y = [Y_0..Y_{N-1}]_W                           Eq. 7
 *   chained layers: O^m = I^{m+1}, no communication between patches
 *   stochastic boundaries per minibatch
 *
 * CONVENTIONS (apply to every call)
 *  - Every call returns splitcnn_status_t; nothing throws or exits.  On error
 *    splitcnn_last_error() returns a thread-local message valid until the next
 *    call on the same thread.
 *  - Ownership: the caller owns every device / host buffer (PyTorch allocates
 *    them).  The library owns only splitcnn_plan_t (host memory) and frees it in
 *    splitcnn_plan_destroy().  Compute calls never allocate device memory; the
 *    scratch they need is the caller's `ws` (size from splitcnn_workspace_size).
 *  - Streams: every device call enqueues asynchronously on the given stream and
 *    never synchronises.  CUDA launch errors map to SPLITCNN_ERR_CUDA.
 *  - Levels: a plan over L layers has L+1 activation LEVELS; level m is the
 *    input of layer m, level L the output of the last layer.  At each level the
 *    activations of the split region live in PATCH BUFFERS: patch (i, j)
 *    (row-major, i along H, j along W) is a contiguous [N][Hp_i][Wp_j][Cpad]
 *    array (patch-major NHWC) at element offset
 *        off(i, j) = N * Cpad * (bh[i] * W + (bh[i+1] - bh[i]) * bw[j])
 *    from the level's base pointer, where bh / bw are the level's boundaries.
 *    The whole level occupies N * H * W * Cpad elements.
 *  - Channel padding: Cpad = C rounded up to a multiple of 8.  Padding channels
 *    are written as zero by every producer and must be zero in inputs.
 *  - Weights: [Cout][kh][kw][Cpad_in] in the compute dtype (padding channels
 *    zero).  Bias: float32 [Cout].  Weight / bias gradients: float32, same
 *    layouts.
 *  - Full (unsplit) tensors: logical NCHW, physically NCHW (SPLITCNN_NCHW) or
 *    NHWC with exactly C channels (SPLITCNN_NHWC).
 *  - Sharding: every compute call takes a patch range [p0, p1) in row-major
 *    patch index, so a rank computes only its patches.  The plan is global and
 *    identical on every rank.  p1 = -1 means "all patches".
 *  - Alignment: every device pointer must be 16-byte aligned
 *    (SPLITCNN_ERR_ALIGNMENT otherwise).
 */
#ifndef SPLITCNN_H
#define SPLITCNN_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define SPLITCNN_API __attribute__((visibility("default")))
#else
#define SPLITCNN_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st *splitcnn_stream_t; /* == cudaStream_t */
typedef struct CUevent_st *splitcnn_event_t;   /* == cudaEvent_t  */

typedef enum {
    SPLITCNN_OK = 0,
    SPLITCNN_ERR_INVALID_VALUE = 1,
    SPLITCNN_ERR_ALIGNMENT = 2,
    SPLITCNN_ERR_UNSUPPORTED = 3,
    SPLITCNN_ERR_CUDA = 4,
    SPLITCNN_ERR_OOM = 5
} splitcnn_status_t;

/* Storage / compute precision of activations and weights.  Accumulation is fp32.
 *  BF16: bf16 storage, tcgen05 kind::f16 where the shape allows.
 *  TF32: fp32 storage; forward / stride-1 data gradient as ONE tcgen05 kind::tf32 pass (operands read as
 *        TF32); weight gradient by bf16 operand splitting (v = v1 + v2, products of i + j <= 1) on the
 *        bf16 tensor-core kernels.  Error ~1e-3..1e-4 normwise (R13: held to 2e-3).
 *  FP32: fp32 storage, fp32-accurate (R13: 1e-4): forward (conv_fwd_ws with a workspace) and stride-1
 *        data gradient as 3xTF32 (v = hi + lo; lo*W_hi + hi*W_lo + hi*W_hi, three kind::tf32 passes),
 *        weight gradient by 3-way bf16 splitting (products of i + j <= 2); FFMA on the CUDA cores where
 *        the tensor-core path does not take the shape (and for conv_fwd without a workspace).
 *  All three share the element layout of their storage type; every non-conv op treats TF32 as FP32. */
typedef enum { SPLITCNN_BF16 = 0, SPLITCNN_FP32 = 1, SPLITCNN_TF32 = 2 } splitcnn_dtype_t;

typedef enum { SPLITCNN_OP_CONV = 0, SPLITCNN_OP_MAXPOOL = 1 } splitcnn_op_t;

typedef enum {
    SPLITCNN_NCHW = 0,
    SPLITCNN_NHWC = 1,
    /* split only: NCHW full tensor of C/4 channels and 2H x 2W pixels read space-to-depth by 2:
     * level channel 4c + 2*ph + pw of pixel (h, w) = x[n, c, 2h + ph, 2w + pw].  A stride-2 conv on the
     * full tensor equals a stride-1 conv on this level with regrouped weights (the ResNet stem). */
    SPLITCNN_NCHW_S2D = 2
} splitcnn_layout_t;

/* flags */
#define SPLITCNN_FLAG_RELU 0x1u            /* conv_fwd: fuse ReLU into the epilogue */
#define SPLITCNN_FLAG_POOL_RELU_MASK 0x2u  /* pool_fwd: record [max > 0] in argmax bit 7;
                                              pool_bwd: multiply dX by that bit (the backward
                                              of the ReLU feeding the pool)          */
#define SPLITCNN_FLAG_DGRAD_WEIGHTS 0x4u   /* conv_bwd_data: `w` is the prepared buffer written by
                                              splitcnn_conv_dgrad_weights (no flip inside the call, ws unused);
                                              ERR_INVALID_VALUE where that buffer's size is 0 */
#define SPLITCNN_FLAG_FORCE_SIMT 0x100u    /* conv calls: use the CUDA-core kernels even where
                                              the tcgen05 kernel applies (testing)          */

/* One window-based layer Op(X, k, s, p).  Pads are the UNSPLIT layer's. */
typedef struct {
    int32_t op;          /* splitcnn_op_t */
    int32_t kh, kw;      /* window */
    int32_t sh, sw;      /* stride */
    int32_t ph_b, ph_e;  /* padding along H: begin, end */
    int32_t pw_b, pw_e;  /* padding along W */
    int32_t cin, cout;   /* channels (cin == cout for MAXPOOL) */
} splitcnn_layer_t;

typedef struct splitcnn_plan_s *splitcnn_plan_t;

#define SPLITCNN_MAX_SPLITS 32   /* patches per spatial dimension */

/* Geometry of one activation level (all pointers point into plan-owned memory). */
typedef struct {
    int32_t N, C, Cpad, H, W;
    int32_t n_h, n_w;         /* patch grid */
    const int32_t *bh;        /* n_h + 1 boundaries along H (bh[0] = 0, bh[n_h] = H) */
    const int32_t *bw;        /* n_w + 1 boundaries along W */
    int64_t total_elems;      /* N * H * W * Cpad: elements of the level's patch buffers */
} splitcnn_level_t;

/* Geometry of one layer: per-patch pads (Eq. 5, P:139-141 with the R1 reading). */
typedef struct {
    splitcnn_layer_t layer;
    int32_t n_h, n_w;
    const int32_t *pad_h;     /* 2 * n_h: (begin, end) per patch row    */
    const int32_t *pad_w;     /* 2 * n_w: (begin, end) per patch column */
} splitcnn_layer_geom_t;

/* ------------------------------------------------------------------ errors */
SPLITCNN_API const char *splitcnn_last_error(void);
SPLITCNN_API const char *splitcnn_status_string(splitcnn_status_t s);
SPLITCNN_API const char *splitcnn_version(void);
/* Total number of CUDA kernels this library has launched in the process (instrumentation). */
SPLITCNN_API splitcnn_status_t splitcnn_kernel_launches(uint64_t *count);

/* ------------------------------------------------------------------ boundaries (host) */
/* "As evenly as possible": O[i] = floor(i * L / n), O[n] = L.
 * O has n + 1 entries.  Errors: n < 1, n > L. */
SPLITCNN_API splitcnn_status_t splitcnn_boundaries_even(int32_t L, int32_t n, int32_t *O);

/* Stochastic splitting: one scheme per minibatch `step` and per spatial
 * dimension.  s_0 = 0, s_i ~ DiscreteUniform(ceil((i-w)L/n), floor((i+w)L/n)) for i > 0.
 * RNG: SplitMix64 with state0 = seed ^ (step * 0x9E3779B97F4A7C15); H draws
 * first (i = 1..nh-1), then W; value = lo + next() % (hi - lo + 1); an empty range
 * (lo > hi) takes floor(i L / n) without a draw.  Errors: omega outside [0, 0.5). */
SPLITCNN_API splitcnn_status_t splitcnn_boundaries_random(int32_t Lh, int32_t nh, int32_t Lw, int32_t nw,
                                             double omega, uint64_t seed, uint64_t step,
                                             int32_t *O_h, int32_t *O_w);

/* ------------------------------------------------------------------ plan (host) */
/* Build the chained plan of a split region.  O_h (n_h + 1 entries) and O_w partition the
 * LAST layer's output; each earlier layer's schemes follow backward:
 * I_i = s * O_i (R2, within [lb, ub] of Eq. 1-2 whenever p_b <= k - s), pads from Eq. 5,
 * and O^{m-1} = I^m.  Errors (SPLITCNN_ERR_INVALID_VALUE): O not strictly
 * increasing, O[0] != 0, O[n] != output length, an empty patch at any level, output
 * size <= 0, channel chain mismatch, n_h or n_w > SPLITCNN_MAX_SPLITS. */
SPLITCNN_API splitcnn_status_t splitcnn_plan_create(const splitcnn_layer_t *layers, int32_t nlayers,
                                       int32_t N, int32_t C, int32_t H, int32_t W,
                                       const int32_t *O_h, int32_t n_h,
                                       const int32_t *O_w, int32_t n_w,
                                       splitcnn_plan_t *out);
SPLITCNN_API splitcnn_status_t splitcnn_plan_destroy(splitcnn_plan_t plan);
SPLITCNN_API splitcnn_status_t splitcnn_plan_num_layers(splitcnn_plan_t plan, int32_t *nlayers);
SPLITCNN_API splitcnn_status_t splitcnn_plan_level(splitcnn_plan_t plan, int32_t level, splitcnn_level_t *out);
SPLITCNN_API splitcnn_status_t splitcnn_plan_layer(splitcnn_plan_t plan, int32_t layer, splitcnn_layer_geom_t *out);

/* Scratch bytes needed by a compute call (op: 0 = conv_fwd, 1 = conv_bwd_data,
 * 2 = conv_bwd_filter); 0 when none is needed. */
SPLITCNN_API splitcnn_status_t splitcnn_workspace_size(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                          int32_t op, size_t *bytes);

/* ------------------------------------------------------------------ split / merge */
/* Eq. 4: copy the full tensor x (level `level`'s N, C, H, W; layout x_layout) into
 * the level's patch buffers (+ transpose to NHWC, + zero channel padding).  SPLITCNN_NCHW_S2D needs
 * C % 4 == 0 and even patch boundaries are implied (x is N x C/4 x 2H x 2W). */
SPLITCNN_API splitcnn_status_t splitcnn_split(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                 const void *x, int32_t x_layout, void *patches,
                                 int32_t p0, int32_t p1, splitcnn_stream_t stream);

/* Eq. 7: concatenate the level's patch buffers into the full tensor y. */
/* Space-to-depth(2) split of an NCHW tensor with x_channels channels and 2H x 2W pixels into a level
 * of C >= 4 * x_channels channels: level channel 4c + 2ph + pw of (h, w) = x[n, c, 2h + ph, 2w + pw],
 * channels >= 4 * x_channels are zero (so a stride-2 stem can run as a stride-1 conv on a level padded
 * to a tensor-core-friendly channel count).  Errors: x_channels < 1 or 4 * x_channels > C. */
SPLITCNN_API splitcnn_status_t splitcnn_split_s2d(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                      const void *x, int32_t x_channels, void *patches,
                                      int32_t p0, int32_t p1, splitcnn_stream_t stream);
/* Eq. 4 from a ROW WINDOW of the input: x holds only rows [row0, row1) of the level's logical tensor
 * (NCHW as [N][C][row1 - row0][W], or NHWC as [N][row1 - row0][W][C]) -- e.g. the rows of the patch
 * rows a rank owns under patch-row sharding, so a rank copies only its own input rows to
 * the device.  Same output as splitcnn_split on the full tensor.  Errors: layout not NCHW / NHWC, an
 * empty or out-of-range window, a patch of [p0, p1) with rows outside the window. */
SPLITCNN_API splitcnn_status_t splitcnn_split_rows(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                      const void *x, int32_t x_layout, int32_t row0, int32_t row1,
                                      void *patches, int32_t p0, int32_t p1, splitcnn_stream_t stream);
SPLITCNN_API splitcnn_status_t splitcnn_merge(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                 const void *patches, void *y, int32_t y_layout,
                                 int32_t p0, int32_t p1, splitcnn_stream_t stream);

/* ------------------------------------------------------------------ convolution */
/* Forward, Eq. 6: for every patch in [p0, p1),
 *   Y_p[n,oh,ow,co] = act(bias[co] + sum_{r,c,ci} X~_p[n, oh*sh - pt + r, ow*sw - pl + c, ci] W[co,r,c,ci])
 * with X~_p the patch zero-padded by its own pads (pt, pl = the patch's begin pads).
 * x: level `layer` patches; y: level `layer + 1` patches; bias nullable; flags: RELU.
 * Errors: layer is not a conv. */
SPLITCNN_API splitcnn_status_t splitcnn_conv_fwd(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                    const void *x, const void *w, const float *bias, void *y,
                                    uint32_t flags, int32_t p0, int32_t p1, splitcnn_stream_t stream);

/* The same with a caller workspace (size: splitcnn_workspace_size, op 0): with SPLITCNN_FP32 the forward
 * then runs as 3xTF32 on the tensor cores (the hi / lo operand halves live in ws); without one (or with
 * BF16 / TF32, which need none) it is splitcnn_conv_fwd. */
SPLITCNN_API splitcnn_status_t splitcnn_conv_fwd_ws(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                       const void *x, const void *w, const float *bias, void *y,
                                       uint32_t flags, void *ws, size_t ws_bytes, int32_t p0, int32_t p1,
                                       splitcnn_stream_t stream);

/* Forward with the residual join fused (ResNet basic block): y = act(conv(x) + bias + residual), the
 * residual a level `layer + 1` buffer (same layout as y, must not alias it).  bf16 on the tensor cores: the
 * epilogue loads the residual tile with the accumulator and rounds once; other shapes / precisions run
 * conv_fwd_ws then splitcnn_add (the conv output rounded to the storage type first).  ws as conv_fwd_ws. */
SPLITCNN_API splitcnn_status_t splitcnn_conv_fwd_res(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                        const void *x, const void *w, const float *bias, const void *residual,
                                        void *y, uint32_t flags, void *ws, size_t ws_bytes, int32_t p0, int32_t p1,
                                        splitcnn_stream_t stream);

/* Fused forward of a conv (+bias, ReLU) `layer` and the 2x2 / stride-2 / unpadded max-pool
 * `layer + 1` that follows it (ReLU in place): the tcgen05 epilogue pools the
 * bf16-rounded conv outputs of each tile and writes ONLY the pool's output y_pool (level layer+2
 * patches) and its argmax bytes (same layout as y_pool; window index r*2 + c of the first maximum,
 * bit 7 = [max > 0], exactly as splitcnn_pool_fwd with FLAG_POOL_RELU_MASK).  The conv output
 * (level layer+1) is never materialised: the backward pass needs only the argmax (pool_bwd with
 * FLAG_POOL_RELU_MASK applies the ReLU mask).  Results are bitwise equal to conv_fwd followed by
 * pool_fwd.  Patch-local pool windows never straddle a tile: the pool's I = 2*O (R2) makes every conv
 * output patch extent even.  flags must hold RELU | POOL_RELU_MASK.
 * Errors: ERR_UNSUPPORTED when the pair is not fusable (see splitcnn_conv_pool_supported; callers
 * then run conv_fwd + pool_fwd). */
SPLITCNN_API splitcnn_status_t splitcnn_conv_pool_fwd(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                         const void *x, const void *w, const float *bias, void *y_pool,
                                         uint8_t *argmax, uint32_t flags, int32_t p0, int32_t p1,
                                         splitcnn_stream_t stream);
/* *supported = 1 when splitcnn_conv_pool_fwd takes (layer, layer + 1) for dtype: BF16, a conv on the
 * tcgen05 path other than the 8-channel-input one, Cout a multiple of 16 equal to its channel pad,
 * followed by a 2x2 / stride-2 max-pool with zero pads. */
SPLITCNN_API splitcnn_status_t splitcnn_conv_pool_supported(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                               int32_t *supported);

/* Data gradient (adjoint of Eq. 6 within each patch):
 *   dX_p[n,h,w,ci] = sum over co, r, c with oh = (h + pt - r)/sh integral and in range
 *                    of dY_p[n,oh,ow,co] W[co,r,c,ci],   then * [relu_src > 0] if relu_src.
 * dy: level layer+1; dx, relu_src (nullable): level `layer`.  ws: splitcnn_workspace_size(op=1).
 * BF16 runs on tcgen05: stride 1 as the forward kernel with 180-degree-rotated weights, stride 2 by
 * output phase (S*S stride-1 correlations with tap subsets written through strided dX views; phases
 * no tap reaches, k < s, are zero-filled). */
SPLITCNN_API splitcnn_status_t splitcnn_conv_bwd_data(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                         const void *dy, const void *w, void *dx, const void *relu_src,
                                         void *ws, size_t ws_bytes, uint32_t flags,
                                         int32_t p0, int32_t p1, splitcnn_stream_t stream);

/* Dgrad-ready weights, built once per weight version instead of inside every conv_bwd_data call (e.g. on a
 * side stream during the forward pass, off the backward's critical path).  Same arithmetic as the flip the
 * data gradient does in its workspace (the adjoint of Eq. 6): stride 1 the 180-degree-
 * rotated, Cin<->Cout-transposed filter W'[ci][r'][c'][co] = W[co][kh-1-r'][kw-1-c'][ci] (0 for co >= Cout);
 * stride S one sub-filter per output phase that a tap reaches, 1 KB-aligned one after another.
 * _size: bytes of that buffer for (layer, dtype) -- 0 where the data gradient takes none (non-BF16 dtypes,
 * the CUDA-core path); then conv_bwd_data must not get FLAG_DGRAD_WEIGHTS.
 * _weights: w = the layer's weights (as conv_bwd_data's `w`), wt: device buffer of >= _size bytes, 256-byte
 * aligned, owned by the caller and read by later conv_bwd_data calls with FLAG_DGRAD_WEIGHTS (stream-ordered:
 * the caller orders those calls after this one).  Errors: ERR_UNSUPPORTED if _size is 0, ERR_INVALID_VALUE
 * for null / misaligned pointers or wt_bytes < _size. */
SPLITCNN_API splitcnn_status_t splitcnn_conv_dgrad_weights_size(splitcnn_plan_t plan, int32_t layer,
                                                   splitcnn_dtype_t dtype, size_t *bytes);
SPLITCNN_API splitcnn_status_t splitcnn_conv_dgrad_weights(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                              const void *w, void *wt, size_t wt_bytes, splitcnn_stream_t stream);

/* Weight gradient summed over the patches [p0, p1) and the batch:
 *   dW[co,r,c,ci] = beta * dW + sum_p sum_{n,oh,ow} dY_p[n,oh,ow,co] X~_p[n, oh*sh-pt+r, ow*sw-pl+c, ci]
 *   db[co]        = beta * db + sum_p sum_{n,oh,ow} dY_p[n,oh,ow,co]          (db nullable)
 * beta is 0 (overwrite) or 1 (accumulate).  The summation order is fixed (deterministic
 * run to run).  ws: splitcnn_workspace_size(op=2); ERR_INVALID_VALUE if too small.  With db, the dY
 * column sums run concurrently on a library-owned side stream (event fork after the work already in
 * `stream`, joined back into `stream` before return): stream semantics and graph capture are kept. */
SPLITCNN_API splitcnn_status_t splitcnn_conv_bwd_filter(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                           const void *x, const void *dy, float *dw, float *db,
                                           float beta, void *ws, size_t ws_bytes, uint32_t flags,
                                           int32_t p0, int32_t p1, splitcnn_stream_t stream);

/* ------------------------------------------------------------------ max-pool */
/* Forward (Eq. 6 with Op = max-pool): the max over the in-patch window elements (padding
 * is -inf) and its argmax as uint8 window-local index r*kw + c of the FIRST
 * maximum in row-major window order (R8, R9).  With FLAG_POOL_RELU_MASK bit 7 of the
 * argmax byte holds [max > 0].  x: level layer; y, argmax: level layer+1 ([N][Ho][Wo][Cpad]
 * bytes per patch, same offsets as y).  Errors: kh * kw > 127. */
SPLITCNN_API splitcnn_status_t splitcnn_pool_fwd(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                    const void *x, void *y, uint8_t *argmax, uint32_t flags,
                                    int32_t p0, int32_t p1, splitcnn_stream_t stream);

/* Backward: dX_p[argmax] += dY_p (summed in fp32 when windows overlap, R10); every element of
 * dx is written (no memset needed).  With FLAG_POOL_RELU_MASK, dX is multiplied by bit 7. */
SPLITCNN_API splitcnn_status_t splitcnn_pool_bwd(splitcnn_plan_t plan, int32_t layer, splitcnn_dtype_t dtype,
                                    const void *dy, const uint8_t *argmax, void *dx, uint32_t flags,
                                    int32_t p0, int32_t p1, splitcnn_stream_t stream);

/* ------------------------------------------------------------------ residual add */
/* Pointwise add on the patch buffers of one level (ResNet residual join; the add is split-
 * invariant, so a shortcut and its sibling branch share the level's I and O).  Acts on
 * the contiguous element span of patches [p0, p1) of `level` (patches of a level are stored back
 * to back).  a, b, y, mask: level buffers (same layout); y may alias a or b.
 *   mask == NULL: y = a + b, then max(., 0) with FLAG_RELU            (forward join)
 *   mask != NULL: y = (a + b) * [mask > 0]                          (backward: sum of a fork's
 *                 two gradient contributions times the ReLU mask of the block output mask)
 *   b == NULL (mask required): y = a * [mask > 0]                   (ReLU backward alone, e.g. the
 *                 output gradient of a stack whose last op is a conv with a fused ReLU)
 * Arithmetic in fp32, one rounding to the storage type.  Errors: null a/y, null b without a mask,
 * misalignment,
 * FLAG_RELU together with a mask. */
SPLITCNN_API splitcnn_status_t splitcnn_add(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                const void *a, const void *b, void *y, const void *mask, uint32_t flags,
                                int32_t p0, int32_t p1, splitcnn_stream_t stream);

/* ------------------------------------------------------------------ global average pool */
/* ResNet head (f2): y[n][c] = mean of x[n, c] over the level's logical H x W (every pixel of every
 * patch; a 1x1-split tail level is plain NHWC).  y: [N][Cpad] in the level dtype (pad channels 0).
 * Backward: dx = dy[n][c] / (H W) at every pixel of every patch (every element written).  Fixed-order
 * fp32 sums: bitwise reproducible.  Errors: null pointers, misalignment. */
SPLITCNN_API splitcnn_status_t splitcnn_gap_fwd(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                    const void *x, void *y, splitcnn_stream_t stream);
SPLITCNN_API splitcnn_status_t splitcnn_gap_bwd(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                    const void *dy, void *dx, splitcnn_stream_t stream);

/* ------------------------------------------------------------------ batch normalisation */
/* Whole-tensor BN on a split level.  BN is not a window operator, so
 * Split-CNN keeps it unsplit: its statistics are those of the LOGICAL tensor over all patches,
 * images and pixels (= unsplit training-mode BN), assembled from per-patch partial sums.  Every call
 * acts on the contiguous span of patches [p0, p1) of `level`; under patch sharding each rank passes
 * its span and the caller sums the [2][C] partial sums across ranks (a 2C-float allreduce) before
 * bn_fwd / bn_bwd.  fp32 partials per block, one fixed-order fp64 sum per channel: bitwise
 * reproducible.  ws: scratch of splitcnn_bn_workspace_size bytes (caller-owned).
 *   bn_stats      sums[0][c] = sum x, sums[1][c] = sum x^2
 *   bn_fwd        mean = sums0/count, var = sums1/count - mean^2 (biased), mean_invstd[0][c] = mean,
 *                 mean_invstd[1][c] = 1/sqrt(var + eps); y = gamma*(x-mean)*invstd + beta (FLAG_RELU:
 *                 then max(., 0)); y may alias x.  count = N*H*W of the logical tensor.
 *   bn_bwd_sums   g = dy*[y > 0] (y = the ReLU output; NULL: g = dy), xhat = (x-mean)*invstd;
 *                 t[0][c] = sum g (= dbeta), t[1][c] = sum g*xhat (= dgamma)
 *   bn_bwd        dx = gamma*invstd*(g - t0/count - xhat*t1/count); dx may alias dy.
 * Channel padding (c >= C) of y / dx is written as zero.  Errors: null pointers, Cpad > 2048. */
SPLITCNN_API splitcnn_status_t splitcnn_bn_workspace_size(splitcnn_plan_t plan, int32_t level, size_t *bytes);
SPLITCNN_API splitcnn_status_t splitcnn_bn_stats(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                     const void *x, float *sums, void *ws, size_t ws_bytes,
                                     int32_t p0, int32_t p1, splitcnn_stream_t stream);
SPLITCNN_API splitcnn_status_t splitcnn_bn_fwd(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                   const void *x, const float *sums, double count, const float *gamma,
                                   const float *beta, float eps, float *mean_invstd, void *y, uint32_t flags,
                                   int32_t p0, int32_t p1, splitcnn_stream_t stream);
SPLITCNN_API splitcnn_status_t splitcnn_bn_bwd_sums(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                        const void *dy, const void *x, const void *y, const float *mean_invstd,
                                        float *t, void *ws, size_t ws_bytes, int32_t p0, int32_t p1,
                                        splitcnn_stream_t stream);
SPLITCNN_API splitcnn_status_t splitcnn_bn_bwd(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                   const void *dy, const void *x, const void *y, const float *mean_invstd,
                                   const float *gamma, const float *t, double count, void *dx,
                                   int32_t p0, int32_t p1, splitcnn_stream_t stream);

/* ------------------------------------------------------------------ offload / prefetch */
/* Patch-granular activation offload (HMMS): after `ready` (recorded by the caller
 * on the compute stream after the buffer's last write, moment 1) copy patch `patch` of level
 * `level` (its contiguous [N][Hp][Wp][Cpad] bytes) to host_pinned on mem_stream and record
 * `done` (the caller makes the compute stream wait on `done` before freeing / overwriting,
 * moment 2).  ready / done nullable.  host_pinned must be page-locked (ERR_INVALID_VALUE). */
SPLITCNN_API splitcnn_status_t splitcnn_offload(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                   int32_t patch, const void *dev_patches, void *host_pinned,
                                   splitcnn_event_t ready, splitcnn_stream_t mem_stream,
                                   splitcnn_event_t done);
/* Prefetch (moments 3-4): host_pinned -> the patch's device bytes on mem_stream after `ready`,
 * then record `done` (the compute stream waits on it before the first backward use). */
SPLITCNN_API splitcnn_status_t splitcnn_prefetch(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                    int32_t patch, const void *host_pinned, void *dev_patches,
                                    splitcnn_event_t ready, splitcnn_stream_t mem_stream,
                                    splitcnn_event_t done);
/* Byte size / byte offset of one patch buffer at a level. */
SPLITCNN_API splitcnn_status_t splitcnn_patch_bytes(splitcnn_plan_t plan, int32_t level, splitcnn_dtype_t dtype,
                                       int32_t patch, size_t *offset, size_t *bytes);

/* ------------------------------------------------------------------ offload planning (host) */
/* Algorithm 1 and the reverse prefetch pass, SURVEY R15.
 * Inputs, per serialized forward op t = 0..T-1: op_time_s[t] (profiled seconds),
 * cand_bytes[t] = bytes of the TSO (patch buffer) that becomes offloadable at op t (0: none),
 * bw_bytes_per_s = measured host-link bandwidth.
 * Outputs: offload[t] = 1 if that TSO is offloaded; sync_at[t] = 1 if op t is an
 * "end of offload" point (compute waits for all outstanding offloads, then frees them);
 * for the backward list (op_time_bwd_s, need_bytes[t] = bytes first needed at backward op t),
 * prefetch_start[t] = the backward op index at which the prefetch for need t starts (-1 none).
 * The ratio cap: an offload is skipped if cumulative offloaded bytes would exceed
 * sum(op_time) * bw. */
SPLITCNN_API splitcnn_status_t splitcnn_offload_plan(int32_t T, const double *op_time_s, const int64_t *cand_bytes,
                                        double bw_bytes_per_s, int32_t *offload, int32_t *sync_at);
SPLITCNN_API splitcnn_status_t splitcnn_prefetch_plan(int32_t T, const double *op_time_bwd_s, const int64_t *need_bytes,
                                         double bw_bytes_per_s, int32_t *prefetch_start);

/* ------------------------------------------------------------------ static memory planning */
/* HMMS static memory planning (§4.4): first-fit placement of n tensor storage
 * objects (TSOs) in ONE contiguous pool, walking the serialized op list.  TSO i occupies
 * ceil(bytes[i] / align) * align bytes from op first_use[i] through op last_use[i] inclusive.  At op
 * t, TSOs whose last use is < t are released first (free neighbours coalesce), then the TSOs first
 * used at t are placed, in index order, at the lowest offset of a free hole they fit in; the pool
 * grows at its end otherwise.  Outputs: offsets[i] (multiples of align; 0 for empty TSOs) and
 * *pool_bytes = the high-water mark.  Host-only, O(n * holes).  Errors: null pointers, align not a
 * power of two, negative size, last_use < first_use. */
SPLITCNN_API splitcnn_status_t splitcnn_memplan(int32_t n, const int64_t *bytes, const int32_t *first_use,
                                    const int32_t *last_use, int64_t align, int64_t *offsets,
                                    int64_t *pool_bytes);

#ifdef __cplusplus
}
#endif
#endif /* SPLITCNN_H */

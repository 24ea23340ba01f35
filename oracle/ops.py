"""O2-O10 -- split, per-patch window ops, merge (TEST INFRASTRUCTURE ONLY).

Patches are lists of numpy float64 arrays in the paper's logical NCHW layout,
indexed [i][j] for patch row i (H) and patch column j (W).  The per-patch
operators call the fp64 direct loops in ``csrc/oracle_loops.c``.

    X_0..X_{N-1} = Split_W(X, I)          Eq. 4, P:148   -> split()
    Y_n = Op(X_n, k, s, p_n)              Eq. 6, P:153   -> conv_fwd(), pool_fwd()
    Y = [Y_0 .. Y_{N-1}]_W                Eq. 7, P:156   -> merge()
    backward: the adjoints of Eq. 6 per patch (no inter-patch communication)
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from .plan import LayerPlan, patch_out_len

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "csrc", "oracle_loops.c")
_LIB = os.path.join(_HERE, "_oracle_loops.so")

_dp = ctypes.POINTER(ctypes.c_double)
_ip = ctypes.POINTER(ctypes.c_int)


def build(force: bool = False) -> str:
    """Compile the C loops (gcc, OpenMP, no FP contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-ffp-contract=off",
                               "-o", _LIB, _SRC, "-lm"])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        i = ctypes.c_int
        _lib.oracle_conv_fwd.argtypes = [_dp, _dp, _dp, _dp] + [i] * 14
        _lib.oracle_conv_bwd_data.argtypes = [_dp, _dp, _dp, _dp] + [i] * 13
        _lib.oracle_conv_bwd_filter.argtypes = [_dp, _dp, _dp, _dp] + [i] * 13
        _lib.oracle_pool_fwd.argtypes = [_dp, _dp, _ip] + [i] * 12
        _lib.oracle_pool_bwd.argtypes = [_dp, _ip, _dp] + [i] * 12
    return _lib


def _d(a):
    return None if a is None else a.ctypes.data_as(_dp)


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


# --------------------------------------------------------------------------- Eq. 4 / Eq. 7
def split(X: np.ndarray, Ih: list[int], Iw: list[int]):
    """Eq. 4 applied on H then W (2-D generalisation): X[:, :, I_i:I_{i+1}, J_j:J_{j+1}]."""
    return [[X[:, :, Ih[i]:Ih[i + 1], Iw[j]:Iw[j + 1]].copy() for j in range(len(Iw) - 1)]
            for i in range(len(Ih) - 1)]


def merge(P) -> np.ndarray:
    """Eq. 7: concatenation along W within a patch row, then along H."""
    return np.concatenate([np.concatenate(row, axis=3) for row in P], axis=2)


# --------------------------------------------------------------------------- one patch
def conv_fwd_patch(X, W, b, sh, sw, pads_h, pads_w, relu=False):
    """O3 on one patch: Op(X_n, k, s, p_n) = conv of the zero-padded patch (+bias, +ReLU)."""
    X, W = _f64(X), _f64(W)
    b = None if b is None else _f64(b)
    N, Ci, Hp, Wp = X.shape
    Co, Ci2, kh, kw = W.shape
    assert Ci == Ci2
    Ho = patch_out_len(Hp, kh, sh, *pads_h)
    Wo = patch_out_len(Wp, kw, sw, *pads_w)
    Y = np.empty((N, Co, Ho, Wo))
    lib().oracle_conv_fwd(_d(X), _d(W), _d(b), _d(Y), N, Ci, Hp, Wp, Co, kh, kw, sh, sw,
                          pads_h[0], pads_w[0], Ho, Wo, int(relu))
    return Y


def conv_bwd_data_patch(dY, W, Hp, Wp, sh, sw, pads_h, pads_w, mask=None):
    """O4 on one patch; ``mask`` (the ReLU output feeding this layer) zeroes dX where mask <= 0."""
    dY, W = _f64(dY), _f64(W)
    mask = None if mask is None else _f64(mask)
    N, Co, Ho, Wo = dY.shape
    _, Ci, kh, kw = W.shape
    dX = np.empty((N, Ci, Hp, Wp))
    lib().oracle_conv_bwd_data(_d(dY), _d(W), _d(mask), _d(dX), N, Ci, Hp, Wp, Co, kh, kw, sh, sw,
                               pads_h[0], pads_w[0], Ho, Wo)
    return dX


def conv_bwd_filter_patch(X, dY, kh, kw, sh, sw, pads_h, pads_w):
    """O5 on one patch: returns (dW_p, db_p)."""
    X, dY = _f64(X), _f64(dY)
    N, Ci, Hp, Wp = X.shape
    _, Co, Ho, Wo = dY.shape
    dW = np.empty((Co, Ci, kh, kw))
    db = np.empty((Co,))
    lib().oracle_conv_bwd_filter(_d(X), _d(dY), _d(dW), _d(db), N, Ci, Hp, Wp, Co, kh, kw, sh, sw,
                                 pads_h[0], pads_w[0], Ho, Wo)
    return dW, db


def pool_fwd_patch(X, kh, kw, sh, sw, pads_h, pads_w):
    """O6 on one patch: (Y, argmax window-local r*kw+c, first max in row-major order)."""
    X = _f64(X)
    N, C, Hp, Wp = X.shape
    Ho = patch_out_len(Hp, kh, sh, *pads_h)
    Wo = patch_out_len(Wp, kw, sw, *pads_w)
    Y = np.empty((N, C, Ho, Wo))
    A = np.empty((N, C, Ho, Wo), dtype=np.int32)
    lib().oracle_pool_fwd(_d(X), _d(Y), A.ctypes.data_as(_ip), N, C, Hp, Wp, kh, kw, sh, sw,
                          pads_h[0], pads_w[0], Ho, Wo)
    return Y, A


def pool_bwd_patch(dY, A, Hp, Wp, kh, kw, sh, sw, pads_h, pads_w):
    """O7 on one patch: dX[argmax] += dY."""
    dY = _f64(dY)
    A = np.ascontiguousarray(A, dtype=np.int32)
    N, C, Ho, Wo = dY.shape
    dX = np.empty((N, C, Hp, Wp))
    lib().oracle_pool_bwd(_d(dY), A.ctypes.data_as(_ip), _d(dX), N, C, Hp, Wp, kh, kw, sh, sw,
                          pads_h[0], pads_w[0], Ho, Wo)
    return dX


# --------------------------------------------------------------------------- all patches of a layer
def _grid(lp: LayerPlan):
    return range(len(lp.Ih) - 1), range(len(lp.Iw) - 1)


def conv_fwd(Xp, W, b, lp: LayerPlan, relu=False):
    """Eq. 6 for every patch of the layer."""
    R, C = _grid(lp)
    return [[conv_fwd_patch(Xp[i][j], W, b, lp.sh, lp.sw, lp.pads_h[i], lp.pads_w[j], relu)
             for j in C] for i in R]


def conv_bwd_data(dYp, W, lp: LayerPlan, maskp=None):
    R, C = _grid(lp)
    return [[conv_bwd_data_patch(dYp[i][j], W, lp.Ih[i + 1] - lp.Ih[i], lp.Iw[j + 1] - lp.Iw[j],
                                 lp.sh, lp.sw, lp.pads_h[i], lp.pads_w[j],
                                 None if maskp is None else maskp[i][j])
             for j in C] for i in R]


def conv_bwd_filter(Xp, dYp, lp: LayerPlan):
    """a5: dW = sum over patches (row-major patch order) of the per-patch weight gradients."""
    R, C = _grid(lp)
    dW = db = None
    for i in R:
        for j in C:
            w, b = conv_bwd_filter_patch(Xp[i][j], dYp[i][j], lp.kh, lp.kw, lp.sh, lp.sw,
                                         lp.pads_h[i], lp.pads_w[j])
            dW = w if dW is None else dW + w
            db = b if db is None else db + b
    return dW, db


def pool_fwd(Xp, lp: LayerPlan):
    R, C = _grid(lp)
    out = [[pool_fwd_patch(Xp[i][j], lp.kh, lp.kw, lp.sh, lp.sw, lp.pads_h[i], lp.pads_w[j])
            for j in C] for i in R]
    return [[o[0] for o in row] for row in out], [[o[1] for o in row] for row in out]


def pool_bwd(dYp, Ap, lp: LayerPlan):
    R, C = _grid(lp)
    return [[pool_bwd_patch(dYp[i][j], Ap[i][j], lp.Ih[i + 1] - lp.Ih[i], lp.Iw[j + 1] - lp.Iw[j],
                            lp.kh, lp.kw, lp.sh, lp.sw, lp.pads_h[i], lp.pads_w[j])
             for j in C] for i in R]


def residual_add(Ap, Bp, relu=False):
    """Residual join of a ResNet basic block, per patch: Y_p = A_p + B_p (then ReLU).  The add is
    pointwise, so the shortcut shares its sibling's split scheme (summation)."""
    out = [[Ap[i][j] + Bp[i][j] for j in range(len(row))] for i, row in enumerate(Ap)]
    return [[np.maximum(y, 0.0) for y in row] for row in out] if relu else out


def batch_norm(Xp, gamma, beta, eps=1e-5, relu=False):
    """Whole-tensor BN on a split level (R11; BN is not a window op, so Split-CNN keeps it
    unsplit): per-channel mean and biased variance over the LOGICAL tensor (all patches, images and
    pixels), y = gamma*(x-mean)/sqrt(var+eps) + beta, then ReLU.  Returns (Yp, mean, invstd)."""
    X = merge(Xp)
    mean = X.mean(axis=(0, 2, 3))
    var = ((X - mean[None, :, None, None]) ** 2).mean(axis=(0, 2, 3))
    invstd = 1.0 / np.sqrt(var + eps)
    Y = (X - mean[None, :, None, None]) * (gamma * invstd)[None, :, None, None] + beta[None, :, None, None]
    if relu:
        Y = np.maximum(Y, 0.0)
    return _resplit(Y, Xp), mean, invstd


def batch_norm_bwd(dYp, Xp, Yp, gamma, mean, invstd, relu=False):
    """Adjoint of batch_norm (training mode): with g = dY*[Y>0] (ReLU) and xhat = (x-mean)*invstd,
    dgamma = sum g*xhat, dbeta = sum g, dX = gamma*invstd*(g - mean(g) - xhat*mean(g*xhat))."""
    dY, X = merge(dYp), merge(Xp)
    g = np.where(merge(Yp) > 0, dY, 0.0) if relu else dY
    xh = (X - mean[None, :, None, None]) * invstd[None, :, None, None]
    M = X.shape[0] * X.shape[2] * X.shape[3]
    dbeta = g.sum(axis=(0, 2, 3))
    dgamma = (g * xh).sum(axis=(0, 2, 3))
    dX = (gamma * invstd)[None, :, None, None] * (g - dbeta[None, :, None, None] / M
                                                 - xh * dgamma[None, :, None, None] / M)
    return _resplit(dX, Xp), dgamma, dbeta


def _resplit(Y, like):
    """Cut a full tensor along the partition of the patch list ``like`` (layout glue)."""
    hs = np.cumsum([0] + [row[0].shape[2] for row in like])
    ws = np.cumsum([0] + [p.shape[3] for p in like[0]])
    return [[Y[:, :, hs[i]:hs[i + 1], ws[j]:ws[j + 1]] for j in range(len(like[0]))] for i in range(len(like))]


def global_avg_pool(Y):
    """ResNet head: mean over the spatial dims of a full NCHW tensor -> [N][C]."""
    return np.asarray(Y).mean(axis=(2, 3))


def global_avg_pool_bwd(G, H, W):
    """Adjoint of global_avg_pool: G[n][c] / (H W) at every pixel."""
    return np.repeat(np.repeat((np.asarray(G) / (H * W))[:, :, None, None], H, axis=2), W, axis=3)


def relu_mask(dXp, Mp):
    """ReLU backward: keep the gradient where the ReLU output is > 0."""
    return [[np.where(Mp[i][j] > 0, dXp[i][j], 0.0) for j in range(len(row))]
            for i, row in enumerate(dXp)]


def argmax_to_plane_index(A, lp: LayerPlan, i: int, j: int):
    """R8: map the window-local argmax of patch (i, j) to torch's global plane index
    h_g * W + w_g of the unsplit input (used by tests for the bit-exact comparison)."""
    N, C, Ho, Wo = A.shape
    oh = np.arange(Ho)[:, None]
    ow = np.arange(Wo)[None, :]
    h = oh * lp.sh - lp.pads_h[i][0] + A // lp.kw + lp.Ih[i]
    w = ow * lp.sw - lp.pads_w[j][0] + A % lp.kw + lp.Iw[j]
    return h * lp.W_in + w


# --------------------------------------------------------------------------- O9 / O10
def offload_roundtrip(buf: np.ndarray) -> np.ndarray:
    """O9: offload then prefetch is the identity on bytes."""
    return buf.copy()


def allreduce_sum(parts):
    """O10: the weight-gradient allreduce is the sum of the per-rank partial sums."""
    out = None
    for p in parts:
        out = np.array(p, dtype=np.float64) if out is None else out + p
    return out

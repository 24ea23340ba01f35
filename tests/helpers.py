"""Test-side marshalling between the oracle's NCHW patches and the library's patch buffers.
(Pure layout glue: slicing, transposes and zero channel padding; no arithmetic of the method.)"""
from __future__ import annotations

import numpy as np


def pack_level(X_nchw: np.ndarray, level: dict) -> np.ndarray:
    """Full NCHW tensor -> flat patch-major NHWC buffer of a level (Cpad zero-padded)."""
    N, C, H, W = X_nchw.shape
    Cp = level["Cpad"]
    out = np.zeros(level["total_elems"], dtype=np.float64)
    bh, bw = level["bh"], level["bw"]
    for i in range(level["n_h"]):
        hp = bh[i + 1] - bh[i]
        for j in range(level["n_w"]):
            wp = bw[j + 1] - bw[j]
            off = N * Cp * (bh[i] * W + hp * bw[j])
            blk = np.zeros((N, hp, wp, Cp))
            blk[..., :C] = X_nchw[:, :, bh[i]:bh[i + 1], bw[j]:bw[j + 1]].transpose(0, 2, 3, 1)
            out[off:off + blk.size] = blk.reshape(-1)
    return out


def pack_patches(P, level: dict) -> np.ndarray:
    """Oracle patch list [i][j] of NCHW arrays -> flat level buffer."""
    return pack_level(merge(P), level)


def unpack_level(buf: np.ndarray, level: dict, keep_pad: bool = False):
    """Flat level buffer -> list [i][j] of NCHW patches (float64)."""
    N, C, Cp, W = level["N"], level["C"], level["Cpad"], level["W"]
    bh, bw = level["bh"], level["bw"]
    buf = np.asarray(buf)
    rows = []
    for i in range(level["n_h"]):
        hp = bh[i + 1] - bh[i]
        row = []
        for j in range(level["n_w"]):
            wp = bw[j + 1] - bw[j]
            off = N * Cp * (bh[i] * W + hp * bw[j])
            blk = buf[off:off + N * hp * wp * Cp].reshape(N, hp, wp, Cp).astype(np.float64)
            row.append(blk.transpose(0, 3, 1, 2)[:, :(Cp if keep_pad else C)])
        rows.append(row)
    return rows


def merge(P):
    return np.concatenate([np.concatenate(r, axis=3) for r in P], axis=2)


def normwise(got: np.ndarray, ref: np.ndarray) -> float:
    """||y - y*||_inf / ||y*||_inf."""
    den = np.abs(ref).max()
    return float(np.abs(got - ref).max() / (den if den > 0 else 1.0))


def w_oihw_to_lib(W: np.ndarray, cpad: int) -> np.ndarray:
    co, ci, kh, kw = W.shape
    out = np.zeros((co, kh, kw, cpad))
    out[..., :ci] = W.transpose(0, 2, 3, 1)
    return out


def w_lib_to_oihw(Wl: np.ndarray, ci: int) -> np.ndarray:
    return np.asarray(Wl)[..., :ci].transpose(0, 3, 1, 2)

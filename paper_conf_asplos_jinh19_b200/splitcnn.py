"""Thin ctypes binding of libsplitcnn.so (include/splitcnn.h) -- argument marshalling only.

Every function has the C name and forwards to the library; tensors are passed as
raw device / host pointers (``tensor.data_ptr()``), streams as ``cudaStream_t``.
There is no fallback: if the shared library is missing this module raises on import.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libsplitcnn.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is not built; run `python -c 'import __graft_entry__ as g; g.build()'` "
                      "(there is no CPU fallback for the split operators)")

_lib = ctypes.CDLL(LIB_PATH)

# ---------------------------------------------------------------- constants (splitcnn.h)
OK, ERR_INVALID_VALUE, ERR_ALIGNMENT, ERR_UNSUPPORTED, ERR_CUDA, ERR_OOM = range(6)
BF16, FP32, TF32 = 0, 1, 2
OP_CONV, OP_MAXPOOL = 0, 1
NCHW, NHWC, NCHW_S2D = 0, 1, 2
FLAG_RELU = 0x1
FLAG_POOL_RELU_MASK = 0x2
FLAG_DGRAD_WEIGHTS = 0x4
FLAG_FORCE_SIMT = 0x100
MAX_SPLITS = 32

EXPORTED = [
    "splitcnn_last_error", "splitcnn_status_string", "splitcnn_version", "splitcnn_kernel_launches",
    "splitcnn_boundaries_even", "splitcnn_boundaries_random",
    "splitcnn_plan_create", "splitcnn_plan_destroy", "splitcnn_plan_num_layers", "splitcnn_plan_level",
    "splitcnn_plan_layer", "splitcnn_workspace_size",
    "splitcnn_split", "splitcnn_split_s2d", "splitcnn_split_rows", "splitcnn_merge",
    "splitcnn_conv_fwd", "splitcnn_conv_fwd_ws", "splitcnn_conv_fwd_res", "splitcnn_conv_bwd_data", "splitcnn_conv_bwd_filter",
    "splitcnn_conv_dgrad_weights_size", "splitcnn_conv_dgrad_weights",
    "splitcnn_pool_fwd", "splitcnn_pool_bwd", "splitcnn_conv_pool_fwd", "splitcnn_conv_pool_supported", "splitcnn_add",
    "splitcnn_gap_fwd", "splitcnn_gap_bwd",
    "splitcnn_bn_workspace_size", "splitcnn_bn_stats", "splitcnn_bn_fwd", "splitcnn_bn_bwd_sums", "splitcnn_bn_bwd",
    "splitcnn_offload", "splitcnn_prefetch", "splitcnn_patch_bytes",
    "splitcnn_offload_plan", "splitcnn_prefetch_plan", "splitcnn_memplan",
]


class Layer(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in
                ("op", "kh", "kw", "sh", "sw", "ph_b", "ph_e", "pw_b", "pw_e", "cin", "cout")]


class LevelInfo(ctypes.Structure):
    _fields_ = [("N", ctypes.c_int32), ("C", ctypes.c_int32), ("Cpad", ctypes.c_int32),
                ("H", ctypes.c_int32), ("W", ctypes.c_int32), ("n_h", ctypes.c_int32), ("n_w", ctypes.c_int32),
                ("bh", ctypes.POINTER(ctypes.c_int32)), ("bw", ctypes.POINTER(ctypes.c_int32)),
                ("total_elems", ctypes.c_int64)]


class LayerGeom(ctypes.Structure):
    _fields_ = [("layer", Layer), ("n_h", ctypes.c_int32), ("n_w", ctypes.c_int32),
                ("pad_h", ctypes.POINTER(ctypes.c_int32)), ("pad_w", ctypes.POINTER(ctypes.c_int32))]


_i32, _u32, _i64, _u64 = ctypes.c_int32, ctypes.c_uint32, ctypes.c_int64, ctypes.c_uint64
_vp, _f32, _f64, _sz = ctypes.c_void_p, ctypes.c_float, ctypes.c_double, ctypes.c_size_t
_pi32 = ctypes.POINTER(ctypes.c_int32)


def _sig(name, args, res=ctypes.c_int):
    f = getattr(_lib, name)
    f.argtypes = args
    f.restype = res


_sig("splitcnn_last_error", [], ctypes.c_char_p)
_sig("splitcnn_status_string", [ctypes.c_int], ctypes.c_char_p)
_sig("splitcnn_version", [], ctypes.c_char_p)
_sig("splitcnn_kernel_launches", [ctypes.POINTER(ctypes.c_uint64)])
_sig("splitcnn_boundaries_even", [_i32, _i32, _pi32])
_sig("splitcnn_boundaries_random", [_i32, _i32, _i32, _i32, _f64, _u64, _u64, _pi32, _pi32])
_sig("splitcnn_plan_create", [ctypes.POINTER(Layer), _i32, _i32, _i32, _i32, _i32, _pi32, _i32, _pi32, _i32,
                              ctypes.POINTER(_vp)])
_sig("splitcnn_plan_destroy", [_vp])
_sig("splitcnn_plan_num_layers", [_vp, _pi32])
_sig("splitcnn_plan_level", [_vp, _i32, ctypes.POINTER(LevelInfo)])
_sig("splitcnn_plan_layer", [_vp, _i32, ctypes.POINTER(LayerGeom)])
_sig("splitcnn_workspace_size", [_vp, _i32, ctypes.c_int, _i32, ctypes.POINTER(_sz)])
_sig("splitcnn_split", [_vp, _i32, ctypes.c_int, _vp, _i32, _vp, _i32, _i32, _vp])
_sig("splitcnn_split_s2d", [_vp, _i32, ctypes.c_int, _vp, _i32, _vp, _i32, _i32, _vp])
_sig("splitcnn_split_rows", [_vp, _i32, ctypes.c_int, _vp, _i32, _i32, _i32, _vp, _i32, _i32, _vp])
_sig("splitcnn_merge", [_vp, _i32, ctypes.c_int, _vp, _vp, _i32, _i32, _i32, _vp])
_sig("splitcnn_conv_fwd", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp, _vp, _u32, _i32, _i32, _vp])
_sig("splitcnn_conv_fwd_ws", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp, _vp, _u32, _vp, _sz, _i32, _i32, _vp])
_sig("splitcnn_conv_fwd_res", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp, _vp, _vp, _u32, _vp, _sz, _i32, _i32, _vp])
_sig("splitcnn_conv_bwd_data", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp, _vp, _vp, _sz, _u32, _i32, _i32, _vp])
_sig("splitcnn_conv_dgrad_weights_size", [_vp, _i32, ctypes.c_int, ctypes.POINTER(_sz)])
_sig("splitcnn_conv_dgrad_weights", [_vp, _i32, ctypes.c_int, _vp, _vp, _sz, _vp])
_sig("splitcnn_conv_bwd_filter", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp, _vp, _f32, _vp, _sz, _u32, _i32, _i32, _vp])
_sig("splitcnn_pool_fwd", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp, _u32, _i32, _i32, _vp])
_sig("splitcnn_pool_bwd", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp, _u32, _i32, _i32, _vp])
_sig("splitcnn_conv_pool_fwd", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp, _vp, _vp, _u32, _i32, _i32, _vp])
_sig("splitcnn_gap_fwd", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp])
_sig("splitcnn_gap_bwd", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp])
_sig("splitcnn_bn_workspace_size", [_vp, _i32, ctypes.POINTER(_sz)])
_sig("splitcnn_bn_stats", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp, _sz, _i32, _i32, _vp])
_sig("splitcnn_bn_fwd", [_vp, _i32, ctypes.c_int, _vp, _vp, _f64, _vp, _vp, _f32, _vp, _vp, _u32, _i32, _i32, _vp])
_sig("splitcnn_bn_bwd_sums", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp, _vp, _vp, _vp, _sz, _i32, _i32, _vp])
_sig("splitcnn_bn_bwd", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp, _vp, _vp, _vp, _f64, _vp, _i32, _i32, _vp])
_sig("splitcnn_add", [_vp, _i32, ctypes.c_int, _vp, _vp, _vp, _vp, _u32, _i32, _i32, _vp])
_sig("splitcnn_conv_pool_supported", [_vp, _i32, ctypes.c_int, _pi32])
_sig("splitcnn_offload", [_vp, _i32, ctypes.c_int, _i32, _vp, _vp, _vp, _vp, _vp])
_sig("splitcnn_prefetch", [_vp, _i32, ctypes.c_int, _i32, _vp, _vp, _vp, _vp, _vp])
_sig("splitcnn_patch_bytes", [_vp, _i32, ctypes.c_int, _i32, ctypes.POINTER(_sz), ctypes.POINTER(_sz)])
_sig("splitcnn_offload_plan", [_i32, ctypes.POINTER(_f64), ctypes.POINTER(_i64), _f64, _pi32, _pi32])
_sig("splitcnn_memplan", [_i32, ctypes.POINTER(_i64), _pi32, _pi32, _i64, ctypes.POINTER(_i64), ctypes.POINTER(_i64)])
_sig("splitcnn_prefetch_plan", [_i32, ctypes.POINTER(_f64), ctypes.POINTER(_i64), _f64, _pi32])


class SplitCNNError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"splitcnn status {status}: {msg}")
        self.status = status


def _check(status: int):
    if status != OK:
        raise SplitCNNError(status, _lib.splitcnn_last_error().decode())


def _ptr(t) -> int | None:
    if t is None:
        return None
    if isinstance(t, int):
        return t
    return t.data_ptr()


def _f32(t) -> int | None:
    """float* argument: a torch tensor must be float32 (the C side reads / writes fp32)."""
    if t is not None and not isinstance(t, int) and getattr(t, "dtype", None) is not None:
        import torch
        if t.dtype != torch.float32:
            raise TypeError(f"expected a float32 tensor, got {t.dtype}")
    return _ptr(t)


def _stream(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _arr(vals, ctype=ctypes.c_int32):
    return (ctype * len(vals))(*vals)


# ---------------------------------------------------------------- host calls
def splitcnn_version() -> str:
    return _lib.splitcnn_version().decode()


def splitcnn_kernel_launches() -> int:
    n = ctypes.c_uint64()
    _check(_lib.splitcnn_kernel_launches(ctypes.byref(n)))
    return n.value


def splitcnn_boundaries_even(L: int, n: int) -> list[int]:
    O = (ctypes.c_int32 * (n + 1))()
    _check(_lib.splitcnn_boundaries_even(L, n, O))
    return list(O)


def splitcnn_boundaries_random(Lh, nh, Lw, nw, omega, seed, step):
    Oh = (ctypes.c_int32 * (nh + 1))()
    Ow = (ctypes.c_int32 * (nw + 1))()
    _check(_lib.splitcnn_boundaries_random(Lh, nh, Lw, nw, float(omega), seed, step, Oh, Ow))
    return list(Oh), list(Ow)


def make_layer(d: dict) -> Layer:
    return Layer(OP_CONV if d["op"] == "conv" else OP_MAXPOOL, d["kh"], d["kw"], d["sh"], d["sw"],
                 d["ph_b"], d["ph_e"], d["pw_b"], d["pw_e"], d["cin"], d["cout"])


def splitcnn_plan_create(layers: list[dict], N, C, H, W, O_h, O_w) -> int:
    arr = (Layer * len(layers))(*[make_layer(l) for l in layers])
    h = _vp()
    _check(_lib.splitcnn_plan_create(arr, len(layers), N, C, H, W, _arr(O_h), len(O_h) - 1, _arr(O_w),
                                     len(O_w) - 1, ctypes.byref(h)))
    return h.value


def splitcnn_plan_destroy(plan: int):
    _check(_lib.splitcnn_plan_destroy(plan))


def splitcnn_plan_num_layers(plan: int) -> int:
    n = ctypes.c_int32()
    _check(_lib.splitcnn_plan_num_layers(plan, ctypes.byref(n)))
    return n.value


def splitcnn_plan_level(plan: int, level: int) -> dict:
    li = LevelInfo()
    _check(_lib.splitcnn_plan_level(plan, level, ctypes.byref(li)))
    return dict(N=li.N, C=li.C, Cpad=li.Cpad, H=li.H, W=li.W, n_h=li.n_h, n_w=li.n_w,
                bh=[li.bh[i] for i in range(li.n_h + 1)], bw=[li.bw[j] for j in range(li.n_w + 1)],
                total_elems=li.total_elems)


def splitcnn_plan_layer(plan: int, layer: int) -> dict:
    g = LayerGeom()
    _check(_lib.splitcnn_plan_layer(plan, layer, ctypes.byref(g)))
    L = g.layer
    return dict(op="conv" if L.op == OP_CONV else "maxpool", kh=L.kh, kw=L.kw, sh=L.sh, sw=L.sw,
                cin=L.cin, cout=L.cout,
                pads_h=[(g.pad_h[2 * i], g.pad_h[2 * i + 1]) for i in range(g.n_h)],
                pads_w=[(g.pad_w[2 * j], g.pad_w[2 * j + 1]) for j in range(g.n_w)])


def splitcnn_workspace_size(plan: int, layer: int, dtype: int, op: int) -> int:
    b = _sz()
    _check(_lib.splitcnn_workspace_size(plan, layer, dtype, op, ctypes.byref(b)))
    return b.value


def splitcnn_patch_bytes(plan: int, level: int, dtype: int, patch: int):
    off, b = _sz(), _sz()
    _check(_lib.splitcnn_patch_bytes(plan, level, dtype, patch, ctypes.byref(off), ctypes.byref(b)))
    return off.value, b.value


def splitcnn_offload_plan(op_time_s, cand_bytes, bw):
    T = len(op_time_s)
    off, sync = (ctypes.c_int32 * T)(), (ctypes.c_int32 * T)()
    _check(_lib.splitcnn_offload_plan(T, _arr(op_time_s, ctypes.c_double), _arr(cand_bytes, ctypes.c_int64),
                                      float(bw), off, sync))
    return list(off), list(sync)


def splitcnn_prefetch_plan(op_time_s, need_bytes, bw):
    T = len(op_time_s)
    st = (ctypes.c_int32 * T)()
    _check(_lib.splitcnn_prefetch_plan(T, _arr(op_time_s, ctypes.c_double), _arr(need_bytes, ctypes.c_int64),
                                       float(bw), st))
    return list(st)


# ---------------------------------------------------------------- device calls
def splitcnn_split(plan, level, dtype, x, x_layout, patches, p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_split(plan, level, dtype, _ptr(x), x_layout, _ptr(patches), p0, p1, _stream(stream)))


def splitcnn_merge(plan, level, dtype, patches, y, y_layout, p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_merge(plan, level, dtype, _ptr(patches), _ptr(y), y_layout, p0, p1, _stream(stream)))


def splitcnn_split_rows(plan, level, dtype, x, x_layout, row0, row1, patches, p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_split_rows(plan, level, dtype, _ptr(x), x_layout, row0, row1, _ptr(patches), p0, p1,
                                    _stream(stream)))


def splitcnn_split_s2d(plan, level, dtype, x, x_channels, patches, p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_split_s2d(plan, level, dtype, _ptr(x), x_channels, _ptr(patches), p0, p1, _stream(stream)))


def splitcnn_conv_fwd(plan, layer, dtype, x, w, bias, y, flags=0, p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_conv_fwd(plan, layer, dtype, _ptr(x), _ptr(w), _f32(bias), _ptr(y), flags, p0, p1,
                                  _stream(stream)))


def splitcnn_conv_fwd_ws(plan, layer, dtype, x, w, bias, y, flags=0, ws=None, ws_bytes=0, p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_conv_fwd_ws(plan, layer, dtype, _ptr(x), _ptr(w), _f32(bias), _ptr(y), flags, _ptr(ws),
                                     ws_bytes, p0, p1, _stream(stream)))


def splitcnn_conv_fwd_res(plan, layer, dtype, x, w, bias, residual, y, flags=0, ws=None, ws_bytes=0, p0=0, p1=-1,
                          stream=None):
    _check(_lib.splitcnn_conv_fwd_res(plan, layer, dtype, _ptr(x), _ptr(w), _f32(bias), _ptr(residual), _ptr(y), flags,
                                      _ptr(ws), ws_bytes, p0, p1, _stream(stream)))


def splitcnn_conv_bwd_data(plan, layer, dtype, dy, w, dx, relu_src=None, ws=None, ws_bytes=0, flags=0, p0=0, p1=-1,
                           stream=None):
    _check(_lib.splitcnn_conv_bwd_data(plan, layer, dtype, _ptr(dy), _ptr(w), _ptr(dx), _ptr(relu_src), _ptr(ws),
                                       ws_bytes, flags, p0, p1, _stream(stream)))


def splitcnn_conv_dgrad_weights_size(plan, layer, dtype) -> int:
    b = _sz(0)
    _check(_lib.splitcnn_conv_dgrad_weights_size(plan, layer, dtype, ctypes.byref(b)))
    return b.value


def splitcnn_conv_dgrad_weights(plan, layer, dtype, w, wt, wt_bytes, stream=None):
    _check(_lib.splitcnn_conv_dgrad_weights(plan, layer, dtype, _ptr(w), _ptr(wt), wt_bytes, _stream(stream)))


def splitcnn_conv_bwd_filter(plan, layer, dtype, x, dy, dw, db=None, beta=0.0, ws=None, ws_bytes=0, flags=0, p0=0,
                             p1=-1, stream=None):
    _check(_lib.splitcnn_conv_bwd_filter(plan, layer, dtype, _ptr(x), _ptr(dy), _f32(dw), _f32(db), float(beta),
                                         _ptr(ws), ws_bytes, flags, p0, p1, _stream(stream)))


def splitcnn_pool_fwd(plan, layer, dtype, x, y, argmax, flags=0, p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_pool_fwd(plan, layer, dtype, _ptr(x), _ptr(y), _ptr(argmax), flags, p0, p1,
                                  _stream(stream)))


def splitcnn_pool_bwd(plan, layer, dtype, dy, argmax, dx, flags=0, p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_pool_bwd(plan, layer, dtype, _ptr(dy), _ptr(argmax), _ptr(dx), flags, p0, p1,
                                  _stream(stream)))


def splitcnn_add(plan, level, dtype, a, b, y, mask=None, flags=0, p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_add(plan, level, dtype, _ptr(a), _ptr(b), _ptr(y), _ptr(mask), flags, p0, p1,
                             _stream(stream)))


def splitcnn_gap_fwd(plan, level, dtype, x, y, stream=None):
    _check(_lib.splitcnn_gap_fwd(plan, level, dtype, _ptr(x), _ptr(y), _stream(stream)))


def splitcnn_gap_bwd(plan, level, dtype, dy, dx, stream=None):
    _check(_lib.splitcnn_gap_bwd(plan, level, dtype, _ptr(dy), _ptr(dx), _stream(stream)))


def splitcnn_bn_workspace_size(plan, level) -> int:
    out = _sz(0)
    _check(_lib.splitcnn_bn_workspace_size(plan, level, ctypes.byref(out)))
    return out.value


def splitcnn_bn_stats(plan, level, dtype, x, sums, ws, ws_bytes, p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_bn_stats(plan, level, dtype, _ptr(x), _f32(sums), _ptr(ws), ws_bytes, p0, p1, _stream(stream)))


def splitcnn_bn_fwd(plan, level, dtype, x, sums, count, gamma, beta, eps, mean_invstd, y, flags=0, p0=0, p1=-1,
                    stream=None):
    _check(_lib.splitcnn_bn_fwd(plan, level, dtype, _ptr(x), _f32(sums), float(count), _f32(gamma), _f32(beta),
                                float(eps), _f32(mean_invstd), _ptr(y), flags, p0, p1, _stream(stream)))


def splitcnn_bn_bwd_sums(plan, level, dtype, dy, x, y, mean_invstd, t, ws, ws_bytes, p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_bn_bwd_sums(plan, level, dtype, _ptr(dy), _ptr(x), _ptr(y), _f32(mean_invstd), _f32(t),
                                     _ptr(ws), ws_bytes, p0, p1, _stream(stream)))


def splitcnn_bn_bwd(plan, level, dtype, dy, x, y, mean_invstd, gamma, t, count, dx, p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_bn_bwd(plan, level, dtype, _ptr(dy), _ptr(x), _ptr(y), _f32(mean_invstd), _f32(gamma),
                                _f32(t), float(count), _ptr(dx), p0, p1, _stream(stream)))


def splitcnn_conv_pool_fwd(plan, layer, dtype, x, w, bias, y_pool, argmax, flags=FLAG_RELU | FLAG_POOL_RELU_MASK,
                           p0=0, p1=-1, stream=None):
    _check(_lib.splitcnn_conv_pool_fwd(plan, layer, dtype, _ptr(x), _ptr(w), _f32(bias), _ptr(y_pool), _ptr(argmax),
                                       flags, p0, p1, _stream(stream)))


def splitcnn_conv_pool_supported(plan, layer, dtype) -> bool:
    out = ctypes.c_int32(0)
    _check(_lib.splitcnn_conv_pool_supported(plan, layer, dtype, ctypes.byref(out)))
    return bool(out.value)


def _ev(e):
    """cudaEvent_t of an int handle or a torch.cuda.Event.  torch creates the CUDA event lazily at the
    first record(); an unrecorded torch event would be a NULL handle, so it is refused here."""
    if e is None:
        return None
    if isinstance(e, int):
        return e
    h = e.cuda_event
    if not h:
        raise ValueError("torch.cuda.Event has no CUDA handle yet (record it once before passing it)")
    return h


def splitcnn_offload(plan, level, dtype, patch, dev_patches, host_pinned, ready=None, mem_stream=None, done=None):
    _check(_lib.splitcnn_offload(plan, level, dtype, patch, _ptr(dev_patches), _ptr(host_pinned), _ev(ready),
                                 _stream(mem_stream), _ev(done)))


def splitcnn_prefetch(plan, level, dtype, patch, host_pinned, dev_patches, ready=None, mem_stream=None, done=None):
    _check(_lib.splitcnn_prefetch(plan, level, dtype, patch, _ptr(host_pinned), _ptr(dev_patches), _ev(ready),
                                  _stream(mem_stream), _ev(done)))


def splitcnn_memplan(nbytes, first_use, last_use, align=256):
    """HMMS static first-fit plan: returns (offsets, pool_bytes)."""
    n = len(nbytes)
    off = (ctypes.c_int64 * max(n, 1))()
    pool = ctypes.c_int64(0)
    _check(_lib.splitcnn_memplan(n, _arr(nbytes, ctypes.c_int64), _arr(first_use), _arr(last_use), align, off,
                                 ctypes.byref(pool)))
    return [off[i] for i in range(n)], pool.value

"""Thin ctypes binding over libdefcon.so (include/defcon.h): same entry-point names,
argument marshalling only.  Every step of the hot path runs in the library's CUDA
kernels; there is no CPU fallback -- if the library is missing or the device cannot
run it, these functions raise.

Tensors are torch CUDA tensors (torch is used for device memory and streams only).
"""
from __future__ import annotations

import ctypes
import os

import torch

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libdefcon.so")

DEFCON_OK, DEFCON_ERR_INVALID_ARG, DEFCON_ERR_UNSUPPORTED, DEFCON_ERR_MISALIGNED, \
    DEFCON_ERR_CUDA, DEFCON_ERR_LIMIT = range(6)
DEFCON_F32, DEFCON_BF16 = 0, 1
DEFCON_SAMPLER_LDG, DEFCON_SAMPLER_TEX, DEFCON_SAMPLER_HYBRID = 0, 1, 2
DEFCON_FP32_3XTF32, DEFCON_FP32_SIMT = 0, 1

# Every symbol include/defcon.h declares (checked by tests/test_abi.py).
EXPORTED = (
    "defcon_offset_dw_conv", "defcon_offset_workspace_size", "defcon_offset_packed_size",
    "defcon_offset_pack_params", "defcon_offset_dw_conv_packed", "defcon_dcn_forward",
    "defcon_dcn_workspace_size", "defcon_deform_columns",
    "defcon_layer_forward_host", "defcon_layer_workspace_size", "defcon_tex_plan_create",
    "defcon_tex_plan_destroy", "defcon_tex_filter_probe", "defcon_status_string",
    "defcon_last_error_detail", "defcon_abi_version",
)

_DTYPES = {torch.float32: DEFCON_F32, torch.bfloat16: DEFCON_BF16}
DEFCON_F16 = 2
_OFF_DTYPES = {torch.float32: DEFCON_F32, torch.float16: DEFCON_F16}   # offsets / mask storage
_SAMPLERS = {"ldg": DEFCON_SAMPLER_LDG, "tex": DEFCON_SAMPLER_TEX, "hybrid": DEFCON_SAMPLER_HYBRID}
_FP32_MODES = {"3xtf32": DEFCON_FP32_3XTF32, "simt": DEFCON_FP32_SIMT}


class DefconError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        self.status = status
        super().__init__(f"{where}: {_status_name(status)} ({detail})")


class defcon_conv_t(ctypes.Structure):
    _fields_ = [("stride_h", ctypes.c_int), ("stride_w", ctypes.c_int),
                ("pad_h", ctypes.c_int), ("pad_w", ctypes.c_int),
                ("dil_h", ctypes.c_int), ("dil_w", ctypes.c_int),
                ("offset_groups", ctypes.c_int),
                ("bound", ctypes.c_int),   # bounded deformation P (R12); 0 = unbounded
                ("offset_dtype", ctypes.c_int)]   # DEFCON_F32 / DEFCON_F16 (tex2D++, R13)


_lib = None


def load_library(path: str = None):
    """Load libdefcon.so; raises if it has not been built (no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    path = path or os.environ.get("DEFCON_LIB") or LIB_PATH   # DEFCON_LIB: dev-probe builds
    if not os.path.exists(path):
        raise RuntimeError(f"{path} not built: run `python -m paper_conf_ipps_jayaweeralwrk24_b200.build`"
                           " (or __graft_entry__.build())")
    lib = ctypes.CDLL(path)
    vp, fp, i, sz = ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int, ctypes.c_size_t
    conv = defcon_conv_t
    lib.defcon_offset_dw_conv.argtypes = [vp, i, i, i, i, i, fp, fp, fp, fp, fp, i, conv, fp, fp, vp,
                                          sz, vp]
    lib.defcon_offset_workspace_size.argtypes = [i, i, i, i, i, conv, ctypes.POINTER(sz)]
    lib.defcon_offset_packed_size.argtypes = [i, i, i, i, ctypes.POINTER(sz)]
    lib.defcon_offset_pack_params.argtypes = [i, i, i, i, fp, fp, fp, fp, vp, sz, vp]
    lib.defcon_offset_dw_conv_packed.argtypes = [vp, i, i, i, i, i, vp, sz, fp, i, conv, fp, fp, vp]
    lib.defcon_dcn_forward.argtypes = [vp, i, i, i, i, fp, fp, vp, fp, i, i, i, conv, i, i, i, vp, vp,
                                       sz, vp, vp]
    lib.defcon_dcn_workspace_size.argtypes = [i, i, i, i, i, i, i, conv, i, i, i,
                                              ctypes.POINTER(sz)]
    lib.defcon_deform_columns.argtypes = [vp, i, i, i, i, fp, fp, i, i, conv, i, vp, vp]
    lib.defcon_layer_forward_host.argtypes = [vp, i, i, i, i, i, fp, fp, fp, fp, fp, vp, fp, i, i,
                                              conv, i, i, i, vp, vp, sz, vp]
    lib.defcon_layer_workspace_size.argtypes = [i, i, i, i, i, i, i, conv, i, i, i,
                                                ctypes.POINTER(sz)]
    lib.defcon_tex_plan_create.argtypes = [i, i, i, i, i, ctypes.POINTER(vp)]
    lib.defcon_tex_plan_destroy.argtypes = [vp]
    lib.defcon_tex_filter_probe.argtypes = [fp, fp, fp, i, vp]
    lib.defcon_status_string.argtypes = [i]
    lib.defcon_status_string.restype = ctypes.c_char_p
    lib.defcon_last_error_detail.restype = ctypes.c_char_p
    for name in EXPORTED:
        if name not in ("defcon_status_string", "defcon_last_error_detail"):
            getattr(lib, name).restype = ctypes.c_int
    _lib = lib
    return lib


def _status_name(status: int) -> str:
    try:
        return load_library().defcon_status_string(status).decode()
    except Exception:
        return str(status)


def _check(rc: int, where: str):
    if rc != DEFCON_OK:
        raise DefconError(rc, where, load_library().defcon_last_error_detail().decode())


def _conv(stride, pad, dil, groups, bound=0, offset_dtype=torch.float32) -> defcon_conv_t:
    s = (stride, stride) if isinstance(stride, int) else tuple(stride)
    p = (pad, pad) if isinstance(pad, int) else tuple(pad)
    d = (dil, dil) if isinstance(dil, int) else tuple(dil)
    if offset_dtype not in _OFF_DTYPES:
        raise ValueError("offsets / mask must be float32 or float16")
    return defcon_conv_t(s[0], s[1], p[0], p[1], d[0], d[1], int(groups), int(bound or 0),
                         _OFF_DTYPES[offset_dtype])


def _out(n, k, s, p, d):
    span = n + 2 * p - d * (k - 1) - 1
    return 0 if span < 0 else span // s + 1


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _dev_tensor(t, name, dtype=None, shape=None, allow_none=False):
    if t is None:
        if allow_none:
            return
        raise ValueError(f"{name} is required")
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    if dtype is not None and t.dtype != dtype:
        raise ValueError(f"{name} must be {dtype}, got {t.dtype}")
    if shape is not None and tuple(t.shape) != tuple(shape):
        raise ValueError(f"{name} shape {tuple(t.shape)} != {tuple(shape)}")


def _stream_handle(stream):
    s = torch.cuda.current_stream() if stream is None else stream
    return ctypes.c_void_p(s.cuda_stream)


def _on(stream):
    """Context that makes `stream` current while this module allocates outputs and scratch:
    the workspace zero-fill is then ordered before the kernel on the same stream, and the
    caching allocator ties the temporaries to that stream (their blocks are not reused by
    another stream while the kernel may still run)."""
    return torch.cuda.stream(stream) if stream is not None else _NullCtx()


class _NullCtx:
    def __enter__(self):
        return self

    def __exit__(self, *exc):
        return False


def defcon_offset_workspace_size(N, H, W, C, K=3, stride=1, pad=1, dil=1, offset_groups=1) -> int:
    lib = load_library()
    out = ctypes.c_size_t(0)
    rc = lib.defcon_offset_workspace_size(N, H, W, C, K, _conv(stride, pad, dil, offset_groups),
                                          ctypes.byref(out))
    _check(rc, "defcon_offset_workspace_size")
    return int(out.value)


def defcon_offset_dw_conv(x, dw_w, dw_scale, dw_shift, pw_w, pw_b=None, K=3, stride=1, pad=1,
                          dil=1, offset_groups=1, with_mask=True, offset=None, mask=None,
                          workspace=None, stream=None, offset_dtype=torch.float32):
    """Step 1: lightweight offset branch.  Returns (offset, mask|None), stored as
    offset_dtype (torch.float16: the 16-bit offsets of tex2D++, R13)."""
    lib = load_library()
    _dev_tensor(x, "x")
    if x.dtype not in _DTYPES:
        raise ValueError("x must be float32 or bfloat16")
    N, H, W, C = x.shape
    cv = _conv(stride, pad, dil, offset_groups, 0, offset_dtype)
    Ho, Wo = _out(H, 3, cv.stride_h, cv.pad_h, cv.dil_h), _out(W, 3, cv.stride_w, cv.pad_w, cv.dil_w)
    G, KK = int(offset_groups), K * K
    OC = G * KK * (3 if with_mask else 2)
    _dev_tensor(dw_w, "dw_w", torch.float32, (C, 3, 3))
    _dev_tensor(dw_scale, "dw_scale", torch.float32, (C,))
    _dev_tensor(dw_shift, "dw_shift", torch.float32, (C,))
    _dev_tensor(pw_w, "pw_w", torch.float32, (OC, C))
    _dev_tensor(pw_b, "pw_b", torch.float32, (OC,), allow_none=True)
    with _on(stream):
        if offset is None:
            offset = torch.empty((N, Ho, Wo, G, KK, 2), device=x.device, dtype=offset_dtype)
        if with_mask and mask is None:
            mask = torch.empty((N, Ho, Wo, G, KK), device=x.device, dtype=offset_dtype)
        if workspace is None:
            workspace = torch.empty(defcon_offset_workspace_size(N, H, W, C, K, stride, pad, dil,
                                                                 offset_groups),
                                    dtype=torch.uint8, device=x.device)
    _dev_tensor(offset, "offset", offset_dtype, (N, Ho, Wo, G, KK, 2))
    if with_mask:
        _dev_tensor(mask, "mask", offset_dtype, (N, Ho, Wo, G, KK))
    else:
        mask = None
    rc = lib.defcon_offset_dw_conv(_ptr(x), N, H, W, C, _DTYPES[x.dtype], _ptr(dw_w), _ptr(dw_scale),
                                   _ptr(dw_shift), _ptr(pw_w), _ptr(pw_b), K, cv, _ptr(offset),
                                   _ptr(mask), _ptr(workspace),
                                   workspace.numel() * workspace.element_size(),
                                   _stream_handle(stream))
    _check(rc, "defcon_offset_dw_conv")
    return offset, mask


def defcon_offset_pack_params(dw_w, dw_scale, dw_shift, pw_w, K=3, offset_groups=1, with_mask=True,
                              packed=None, stream=None):
    """Step 1's parameters packed once per set of weights (include/defcon.h,
    defcon_offset_pack_params); returns the packed uint8 device tensor for
    defcon_offset_dw_conv_packed."""
    lib = load_library()
    C = int(dw_w.shape[0])
    G, KK = int(offset_groups), K * K
    OC = G * KK * (3 if with_mask else 2)
    _dev_tensor(dw_w, "dw_w", torch.float32, (C, 3, 3))
    _dev_tensor(dw_scale, "dw_scale", torch.float32, (C,))
    _dev_tensor(dw_shift, "dw_shift", torch.float32, (C,))
    _dev_tensor(pw_w, "pw_w", torch.float32, (OC, C))
    out = ctypes.c_size_t(0)
    _check(lib.defcon_offset_packed_size(C, K, G, int(with_mask), ctypes.byref(out)), "defcon_offset_packed_size")
    with _on(stream):
        if packed is None:
            packed = torch.empty(int(out.value), dtype=torch.uint8, device=dw_w.device)
    _dev_tensor(packed, "packed")
    rc = lib.defcon_offset_pack_params(C, K, G, int(with_mask), _ptr(dw_w), _ptr(dw_scale), _ptr(dw_shift),
                                       _ptr(pw_w), _ptr(packed), packed.numel() * packed.element_size(),
                                       _stream_handle(stream))
    _check(rc, "defcon_offset_pack_params")
    return packed


def defcon_offset_dw_conv_packed(x, packed, pw_b=None, K=3, stride=1, pad=1, dil=1, offset_groups=1,
                                 with_mask=True, offset=None, mask=None, stream=None,
                                 offset_dtype=torch.float32):
    """Step 1 from pre-packed parameters (defcon_offset_pack_params): the same results as
    defcon_offset_dw_conv without the per-call parameter packing."""
    lib = load_library()
    _dev_tensor(x, "x")
    if x.dtype not in _DTYPES:
        raise ValueError("x must be float32 or bfloat16")
    _dev_tensor(packed, "packed")
    N, H, W, C = x.shape
    cv = _conv(stride, pad, dil, offset_groups, 0, offset_dtype)
    Ho, Wo = _out(H, 3, cv.stride_h, cv.pad_h, cv.dil_h), _out(W, 3, cv.stride_w, cv.pad_w, cv.dil_w)
    G, KK = int(offset_groups), K * K
    OC = G * KK * (3 if with_mask else 2)
    _dev_tensor(pw_b, "pw_b", torch.float32, (OC,), allow_none=True)
    with _on(stream):
        if offset is None:
            offset = torch.empty((N, Ho, Wo, G, KK, 2), device=x.device, dtype=offset_dtype)
        if with_mask and mask is None:
            mask = torch.empty((N, Ho, Wo, G, KK), device=x.device, dtype=offset_dtype)
    _dev_tensor(offset, "offset", offset_dtype, (N, Ho, Wo, G, KK, 2))
    if with_mask:
        _dev_tensor(mask, "mask", offset_dtype, (N, Ho, Wo, G, KK))
    else:
        mask = None
    rc = lib.defcon_offset_dw_conv_packed(_ptr(x), N, H, W, C, _DTYPES[x.dtype], _ptr(packed),
                                          packed.numel() * packed.element_size(), _ptr(pw_b), K, cv,
                                          _ptr(offset), _ptr(mask), _stream_handle(stream))
    _check(rc, "defcon_offset_dw_conv_packed")
    return offset, mask


def defcon_dcn_workspace_size(N, H, W, Cin, Cout, Kh, Kw, stride=1, pad=1, dil=1, offset_groups=1,
                              dtype=torch.bfloat16, sampler="ldg", fp32_mode="simt") -> int:
    lib = load_library()
    out = ctypes.c_size_t(0)
    rc = lib.defcon_dcn_workspace_size(N, H, W, Cin, Cout, Kh, Kw,
                                       _conv(stride, pad, dil, offset_groups), _DTYPES[dtype],
                                       _SAMPLERS[sampler], _FP32_MODES[fp32_mode], ctypes.byref(out))
    _check(rc, "defcon_dcn_workspace_size")
    return int(out.value)


def defcon_dcn_forward(x, offset, mask, weight, bias=None, stride=1, pad=1, dil=1, offset_groups=1,
                       sampler="ldg", fp32_mode="simt", y=None, workspace=None, tex_plan=None,
                       stream=None, bound=0):
    """Step 2 (Eq.2 P:58 + Eq.3): deformable conv forward, NHWC.  Returns y.
    bound = P > 0: bounded deformation (reading R12; the paper's P = 7)."""
    lib = load_library()
    _dev_tensor(x, "x")
    if x.dtype not in _DTYPES:
        raise ValueError("x must be float32 or bfloat16")
    N, H, W, Cin = x.shape
    _dev_tensor(weight, "weight", x.dtype)
    Cout, Kh, Kw, Cw = weight.shape
    if Cw != Cin:
        raise ValueError("weight Cin mismatch")
    odt = offset.dtype if offset is not None else torch.float32   # float16: tex2D++ offsets (R13)
    cv = _conv(stride, pad, dil, offset_groups, bound, odt)
    Ho, Wo = _out(H, Kh, cv.stride_h, cv.pad_h, cv.dil_h), _out(W, Kw, cv.stride_w, cv.pad_w, cv.dil_w)
    G = int(offset_groups)
    _dev_tensor(offset, "offset", odt, (N, Ho, Wo, G, Kh * Kw, 2))
    _dev_tensor(mask, "mask", odt, (N, Ho, Wo, G, Kh * Kw), allow_none=True)
    _dev_tensor(bias, "bias", torch.float32, (Cout,), allow_none=True)
    with _on(stream):
        if y is None:
            y = torch.empty((N, Ho, Wo, Cout), device=x.device, dtype=x.dtype)
        if workspace is None:
            need = defcon_dcn_workspace_size(N, H, W, Cin, Cout, Kh, Kw, stride, pad, dil,
                                             offset_groups, x.dtype, sampler, fp32_mode)
            if need:   # zero before first use, on the stream the kernel runs on
                workspace = torch.zeros(need, dtype=torch.uint8, device=x.device)
    _dev_tensor(y, "y", x.dtype, (N, Ho, Wo, Cout))
    ws_bytes = 0 if workspace is None else workspace.numel() * workspace.element_size()
    plan = None if tex_plan is None else tex_plan.handle
    rc = lib.defcon_dcn_forward(_ptr(x), N, H, W, Cin, _ptr(offset), _ptr(mask), _ptr(weight),
                                _ptr(bias), Cout, Kh, Kw, cv, _DTYPES[x.dtype], _SAMPLERS[sampler],
                                _FP32_MODES[fp32_mode], _ptr(y), _ptr(workspace), ws_bytes, plan,
                                _stream_handle(stream))
    _check(rc, "defcon_dcn_forward")
    return y


def defcon_deform_columns(x, offset, mask, K=3, stride=1, pad=1, dil=1, offset_groups=1, columns=None,
                          stream=None, bound=0):
    """Sampling step alone (Eq.3 P:63-67 + mask, the "two-step" split P:69-76): returns the
    deformable columns [N*Ho*Wo, K*K*Cin] in x's dtype."""
    lib = load_library()
    _dev_tensor(x, "x")
    if x.dtype not in _DTYPES:
        raise ValueError("x must be float32 or bfloat16")
    N, H, W, Cin = x.shape
    Kh, Kw = (K, K) if isinstance(K, int) else K
    odt = offset.dtype if offset is not None else torch.float32
    cv = _conv(stride, pad, dil, offset_groups, bound, odt)
    Ho, Wo = _out(H, Kh, cv.stride_h, cv.pad_h, cv.dil_h), _out(W, Kw, cv.stride_w, cv.pad_w, cv.dil_w)
    G = int(offset_groups)
    _dev_tensor(offset, "offset", odt, (N, Ho, Wo, G, Kh * Kw, 2))
    _dev_tensor(mask, "mask", odt, (N, Ho, Wo, G, Kh * Kw), allow_none=True)
    if columns is None:
        with _on(stream):
            columns = torch.empty((N * Ho * Wo, Kh * Kw * Cin), device=x.device, dtype=x.dtype)
    _dev_tensor(columns, "columns", x.dtype, (N * Ho * Wo, Kh * Kw * Cin))
    rc = lib.defcon_deform_columns(_ptr(x), N, H, W, Cin, _ptr(offset), _ptr(mask), Kh, Kw, cv,
                                   _DTYPES[x.dtype], _ptr(columns), _stream_handle(stream))
    _check(rc, "defcon_deform_columns")
    return columns


def defcon_layer_workspace_size(N, H, W, Cin, Cout, K=3, stride=1, pad=1, dil=1, offset_groups=1,
                                dtype=torch.bfloat16, modulated=True, sampler="ldg",
                                fp32_mode="simt", bound=0, offset_dtype=torch.float32) -> int:
    lib = load_library()
    out = ctypes.c_size_t(0)
    rc = lib.defcon_layer_workspace_size(N, H, W, Cin, _DTYPES[dtype], Cout, K,
                                         _conv(stride, pad, dil, offset_groups, bound, offset_dtype),
                                         int(modulated),
                                         _SAMPLERS[sampler], _FP32_MODES[fp32_mode],
                                         ctypes.byref(out))
    _check(rc, "defcon_layer_workspace_size")
    return int(out.value)


def defcon_layer_forward_host(x_host, branch, weight, bias, y_host, dev_workspace, K=3, stride=1,
                              pad=1, dil=1, offset_groups=1, modulated=True, sampler="ldg",
                              fp32_mode="simt", stream=None, bound=0, offset_dtype=torch.float32):
    """Whole layer from pinned host x to pinned host y (H2D, step 1, step 2, D2H, sync).

    branch: dict of device tensors dw_w, dw_scale, dw_shift, pw_w, pw_b (resident weights).
    """
    lib = load_library()
    if x_host.is_cuda or y_host.is_cuda:
        raise ValueError("x_host / y_host must be host tensors (pinned)")
    N, H, W, Cin = x_host.shape
    Cout = weight.shape[0]
    rc = lib.defcon_layer_forward_host(
        _ptr(x_host), N, H, W, Cin, _DTYPES[x_host.dtype], _ptr(branch["dw_w"]),
        _ptr(branch["dw_scale"]), _ptr(branch["dw_shift"]), _ptr(branch["pw_w"]),
        _ptr(branch.get("pw_b")), _ptr(weight), _ptr(bias), Cout, K,
        _conv(stride, pad, dil, offset_groups, bound, offset_dtype), int(modulated), _SAMPLERS[sampler],
        _FP32_MODES[fp32_mode], _ptr(y_host), _ptr(dev_workspace),
        dev_workspace.numel() * dev_workspace.element_size(), _stream_handle(stream))
    _check(rc, "defcon_layer_forward_host")
    return y_host


class TexPlan:
    """Owns a libdefcon texture plan (layered cudaArray + texture object per image)."""

    def __init__(self, N, H, W, Cin, dtype=torch.bfloat16):
        lib = load_library()
        h = ctypes.c_void_p()
        _check(lib.defcon_tex_plan_create(N, H, W, Cin, _DTYPES[dtype], ctypes.byref(h)),
               "defcon_tex_plan_create")
        self.handle = h

    def close(self):
        if self.handle is not None and self.handle.value:
            load_library().defcon_tex_plan_destroy(self.handle)
        self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def defcon_tex_filter_probe(px, py, out=None, stream=None):
    lib = load_library()
    _dev_tensor(px, "px", torch.float32)
    _dev_tensor(py, "py", torch.float32, tuple(px.shape))
    if out is None:
        with _on(stream):
            out = torch.empty_like(px)
    rc = lib.defcon_tex_filter_probe(_ptr(px), _ptr(py), _ptr(out), px.numel(), _stream_handle(stream))
    _check(rc, "defcon_tex_filter_probe")
    return out


def defcon_abi_version() -> int:
    return int(load_library().defcon_abi_version())

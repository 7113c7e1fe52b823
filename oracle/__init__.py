"""fp64 CPU oracle for the DEFCON hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and the ``cpu_baseline`` /
``--impl reference`` legs of ``bench.py`` may import this package.  It shares
no code with the CUDA product path (``paper_conf_ipps_jayaweeralwrk24_b200``)
and never imports it; the product never imports this.

The arithmetic lives in ``defcon_oracle.c`` (plain C99, fp64, OpenMP over
output rows), compiled to ``liboracle.so`` by :func:`build`.  This module only
marshals numpy fp64 arrays through ctypes.

Every function cites PAPER.md lines ("P:n") and the readings R1..R19 listed
in DESIGN.md.  Pins (what each function is checked against, independently of
itself) are in ``tests/test_oracle_pins.py``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "defcon_oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile defcon_oracle.c -> liboracle.so (gcc, -O2, OpenMP, no FP contraction)."""
    with _lock:
        if (not force and os.path.exists(_LIB_PATH)
                and os.path.getmtime(_LIB_PATH) >= os.path.getmtime(_SRC)):
            return _LIB_PATH
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        cmd = ["gcc", "-std=c99", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
               "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"]
        subprocess.run(cmd, check=True)
        os.replace(tmp, _LIB_PATH)
        return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        dp = ctypes.POINTER(ctypes.c_double)
        i = ctypes.c_int
        lib.oracle_dcn_forward_f64.argtypes = [dp, i, i, i, i, dp, dp, dp, dp, i,
                                               i, i, i, i, i, i, i, i, i, dp]
        lib.oracle_dcn_forward_texq_f64.argtypes = [dp, i, i, i, i, dp, dp, dp, dp, i,
                                                    i, i, i, i, i, i, i, i, i, i, dp]
        lib.oracle_dcn_pixels_f64.argtypes = [dp, i, i, i, i, dp, dp, dp, dp, i,
                                              i, i, i, i, i, i, i, i, i,
                                              ctypes.POINTER(ctypes.c_int64), i, dp]
        lib.oracle_dcn_pixels_texq_f64.argtypes = [dp, i, i, i, i, dp, dp, dp, dp, i,
                                                   i, i, i, i, i, i, i, i, i, i,
                                                   ctypes.POINTER(ctypes.c_int64), i, dp]
        lib.oracle_deform_columns_f64.argtypes = [dp, i, i, i, i, dp, dp, i, i, i, i, i, i, i, i, i,
                                                  ctypes.POINTER(ctypes.c_int64), ctypes.c_long, dp]
        lib.oracle_offset_branch_f64.argtypes = [dp, i, i, i, i, dp, dp, dp, dp, dp,
                                                 i, i, i, i, i, i, dp, dp]
        lib.oracle_bound_offsets_f64.argtypes = [dp, ctypes.c_long, i, i, i, i, i, i, dp]
        lib.oracle_round_f16_array.argtypes = [dp, ctypes.c_long, dp]
        lib.oracle_bilinear_f64.argtypes = [dp, i, i, ctypes.c_long, ctypes.c_double,
                                            ctypes.c_double]
        lib.oracle_bilinear_f64.restype = ctypes.c_double
        lib.oracle_out_size.argtypes = [i, i, i, i, i]
        lib.oracle_set_num_threads.argtypes = [i]
        lib.oracle_set_num_threads.restype = None
        _lib = lib
    return _lib


def _f64(a):
    if a is None:
        return None
    return np.ascontiguousarray(np.asarray(a, dtype=np.float64))


def _p(a):
    if a is None:
        return None
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def num_threads() -> int:
    return int(_load().oracle_num_threads())


def set_num_threads(n: int) -> None:
    _load().oracle_set_num_threads(int(n))


def out_size(n_in: int, k: int, stride: int, pad: int, dil: int) -> int:
    """Output extent of a regular conv (R3)."""
    return int(_load().oracle_out_size(n_in, k, stride, pad, dil))


def bilinear(plane, py: float, px: float) -> float:
    """Eq.3 on one HxW plane (2-D array), zero outside."""
    a = _f64(plane)
    H, W = a.shape
    return float(_load().oracle_bilinear_f64(_p(a), H, W, 1, float(py), float(px)))


def _dcn_shapes(x, offset, weight, stride, pad, dil, G):
    N, H, W, Cin = x.shape
    Cout, Kh, Kw, Cin_w = weight.shape
    if Cin_w != Cin:
        raise ValueError("weight Cin mismatch")
    sh, sw = stride
    ph, pw = pad
    dh, dw = dil
    Ho = out_size(H, Kh, sh, ph, dh)
    Wo = out_size(W, Kw, sw, pw, dw)
    if offset.shape != (N, Ho, Wo, G, Kh * Kw, 2):
        raise ValueError(f"offset shape {offset.shape} != {(N, Ho, Wo, G, Kh * Kw, 2)}")
    return N, H, W, Cin, Cout, Kh, Kw, sh, sw, ph, pw, dh, dw, Ho, Wo


def _pair(v):
    return (v, v) if isinstance(v, int) else tuple(v)


def dcn_forward(x, offset, weight, bias=None, mask=None, stride=1, pad=1, dil=1, G=1):
    """Deformable conv forward, Eq.2 + Eq.3, DCNv2 mask when given (R6).

    x [N,H,W,Cin], offset [N,Ho,Wo,G,K*K,2] (dy,dx), mask [N,Ho,Wo,G,K*K] or None,
    weight [Cout,Kh,Kw,Cin], bias [Cout] or None.  Returns y [N,Ho,Wo,Cout] fp64.
    """
    x, offset, weight, bias, mask = map(_f64, (x, offset, weight, bias, mask))
    (N, H, W, Cin, Cout, Kh, Kw, sh, sw, ph, pw, dh, dw, Ho, Wo) = _dcn_shapes(
        x, offset, weight, _pair(stride), _pair(pad), _pair(dil), G)
    if mask is not None and mask.shape != (N, Ho, Wo, G, Kh * Kw):
        raise ValueError("mask shape")
    y = np.empty((N, Ho, Wo, Cout), np.float64)
    rc = _load().oracle_dcn_forward_f64(_p(x), N, H, W, Cin, _p(offset), _p(mask), _p(weight),
                                        _p(bias), Cout, Kh, Kw, sh, sw, ph, pw, dh, dw, G, _p(y))
    if rc:
        raise ValueError(f"oracle_dcn_forward_f64 rc={rc}")
    return y


def dcn_forward_texq(x, offset, weight, bias=None, mask=None, stride=1, pad=1, dil=1, G=1,
                     quant="round"):
    """Texture-filter model of the layer (R14): fractions quantised to 1/256 ("round" /
    "trunc"), or "hw": the half4-texel filter as measured on B200 -- fractions and the four
    bilinear weights rounded to 1/256 (ties to even), result rounded to binary16."""
    qm = {"round": 1, "trunc": 2, "hw": 3}[quant]
    x, offset, weight, bias, mask = map(_f64, (x, offset, weight, bias, mask))
    (N, H, W, Cin, Cout, Kh, Kw, sh, sw, ph, pw, dh, dw, Ho, Wo) = _dcn_shapes(
        x, offset, weight, _pair(stride), _pair(pad), _pair(dil), G)
    y = np.empty((N, Ho, Wo, Cout), np.float64)
    rc = _load().oracle_dcn_forward_texq_f64(_p(x), N, H, W, Cin, _p(offset), _p(mask),
                                             _p(weight), _p(bias), Cout, Kh, Kw, sh, sw, ph, pw,
                                             dh, dw, G, qm, _p(y))
    if rc:
        raise ValueError(f"oracle_dcn_forward_texq_f64 rc={rc}")
    return y


def dcn_pixels(x, offset, weight, pix_idx, bias=None, mask=None, stride=1, pad=1, dil=1, G=1,
               quant=None):
    """Same definition as dcn_forward, evaluated at flattened output pixels
    pix_idx[t] = (n*Ho + ho)*Wo + wo.  Returns [len(pix_idx), Cout] fp64.
    quant="round"/"trunc": the texture-filter model (R14) of dcn_forward_texq instead."""
    x, offset, weight, bias, mask = map(_f64, (x, offset, weight, bias, mask))
    (N, H, W, Cin, Cout, Kh, Kw, sh, sw, ph, pw, dh, dw, Ho, Wo) = _dcn_shapes(
        x, offset, weight, _pair(stride), _pair(pad), _pair(dil), G)
    idx = np.ascontiguousarray(np.asarray(pix_idx, dtype=np.int64))
    out = np.empty((idx.size, Cout), np.float64)
    ip = idx.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))
    if quant is None:
        rc = _load().oracle_dcn_pixels_f64(
            _p(x), N, H, W, Cin, _p(offset), _p(mask), _p(weight), _p(bias), Cout, Kh, Kw,
            sh, sw, ph, pw, dh, dw, G, ip, int(idx.size), _p(out))
    else:
        rc = _load().oracle_dcn_pixels_texq_f64(
            _p(x), N, H, W, Cin, _p(offset), _p(mask), _p(weight), _p(bias), Cout, Kh, Kw,
            sh, sw, ph, pw, dh, dw, G, {"round": 1, "trunc": 2, "hw": 3}[quant], ip, int(idx.size), _p(out))
    if rc:
        raise ValueError(f"oracle_dcn_pixels_f64 rc={rc}")
    return out


def deform_columns(x, offset, K, pix_idx=None, mask=None, stride=1, pad=1, dil=1, G=1):
    """Sampling step alone (Eq.3 + mask): the deformable im2col rows.

    Returns cols [n_pix, K*K*Cin] fp64 with cols[t, k*Cin + ci] = m_k * X(p_k) for the
    flattened output pixels pix_idx (all pixels when None); K = (Kh, Kw) or int.
    """
    x, offset, mask = map(_f64, (x, offset, mask))
    Kh, Kw = _pair(K)
    N, H, W, Cin = x.shape
    sh, sw = _pair(stride)
    ph, pw = _pair(pad)
    dh, dw = _pair(dil)
    Ho, Wo = out_size(H, Kh, sh, ph, dh), out_size(W, Kw, sw, pw, dw)
    if offset.shape != (N, Ho, Wo, G, Kh * Kw, 2):
        raise ValueError("offset shape")
    if pix_idx is None:
        pix_idx = np.arange(N * Ho * Wo)
    idx = np.ascontiguousarray(np.asarray(pix_idx, dtype=np.int64))
    out = np.empty((idx.size, Kh * Kw * Cin), np.float64)
    rc = _load().oracle_deform_columns_f64(_p(x), N, H, W, Cin, _p(offset), _p(mask), Kh, Kw, sh, sw,
                                           ph, pw, dh, dw, G,
                                           idx.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                           int(idx.size), _p(out))
    if rc:
        raise ValueError(f"oracle_deform_columns_f64 rc={rc}")
    return out


def offset_branch(x, dw_w, dw_scale, dw_shift, pw_w, pw_b, K=3, G=1, with_mask=True,
                  stride=1, pad=1, dil=1):
    """Lightweight offset branch (R10, R11).

    x [N,H,W,C]; dw_w [C,3,3]; dw_scale/dw_shift [C] (folded BN);
    pw_w [OC,C], pw_b [OC] or None, OC = G*K*K*(3 if with_mask else 2).
    Returns (offset [N,Ho,Wo,G,K*K,2], mask [N,Ho,Wo,G,K*K] or None).
    """
    x, dw_w, dw_scale, dw_shift, pw_w, pw_b = map(_f64, (x, dw_w, dw_scale, dw_shift, pw_w, pw_b))
    N, H, W, C = x.shape
    KK = K * K
    OC = G * KK * (3 if with_mask else 2)
    if dw_w.shape != (C, 3, 3) or pw_w.shape != (OC, C):
        raise ValueError("offset-branch weight shapes")
    Ho = out_size(H, 3, stride, pad, dil)
    Wo = out_size(W, 3, stride, pad, dil)
    off = np.empty((N, Ho, Wo, G, KK, 2), np.float64)
    msk = np.empty((N, Ho, Wo, G, KK), np.float64) if with_mask else None
    rc = _load().oracle_offset_branch_f64(_p(x), N, H, W, C, _p(dw_w), _p(dw_scale),
                                          _p(dw_shift), _p(pw_w), _p(pw_b), K, G,
                                          1 if with_mask else 0, stride, pad, dil,
                                          _p(off), _p(msk))
    if rc:
        raise ValueError(f"oracle_offset_branch_f64 rc={rc}")
    return off, msk


def bound_offsets(offset, P, K=3, dil=1):
    """Bounded deformation (section III-A-c; reading R12): each offset restricted so the
    sampling point of tap (i, j) stays in the P x P window centred on the output pixel's centre
    tap (P = 7 in the paper, Fig. 5).  P <= 0 (or None): unbounded, offsets returned as is.

    offset [..., G, Kh*Kw, 2] (dy, dx); K = (Kh, Kw) or int; dil = (dh, dw) or int.
    Returns the bounded offsets (fp64, same shape); feed them to dcn_forward / dcn_pixels.
    """
    off = _f64(offset)
    Kh, Kw = _pair(K)
    dh, dw = _pair(dil)
    if off.shape[-1] != 2 or off.shape[-2] != Kh * Kw:
        raise ValueError("offset shape")
    G = off.shape[-3]
    n_pix = int(np.prod(off.shape[:-3]))
    out = np.empty_like(off)
    rc = _load().oracle_bound_offsets_f64(_p(off), n_pix, G, Kh, Kw, dh, dw, int(P or 0), _p(out))
    if rc:
        raise ValueError(f"oracle_bound_offsets_f64 rc={rc}")
    return out


def round_f16(a):
    """tex2D++ (reading R13): offsets / mask as stored in 16 bits (IEEE binary16, round to
    nearest even), returned as fp64 -- the values a 16-bit-offset DCN computes its coordinates from.
    None passes through."""
    if a is None:
        return None
    a = _f64(a)
    out = np.empty_like(a)
    _load().oracle_round_f16_array(_p(a), int(a.size), _p(out))
    return out

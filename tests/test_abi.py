"""C-ABI contract tests that need no GPU (tier T1).

The library is built (nvcc cross-compiles sm_100a here) and loaded; every symbol
include/defcon.h declares must be exported, and invalid arguments must come back as
the documented status codes *before* any CUDA call (fake device pointers are fine).
"""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ipps_jayaweeralwrk24_b200 import build, _binding
    build.build()
    return _binding.load_library()


def header_symbols():
    txt = open(os.path.join(ROOT, "include", "defcon.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(defcon_[a-z0-9_]+)\s*\(", txt)))


def test_header_symbols_exported(lib):
    from paper_conf_ipps_jayaweeralwrk24_b200 import _binding
    syms = header_symbols()
    assert len(syms) >= 11
    for s in syms:
        assert hasattr(lib, s), s
    assert sorted(_binding.EXPORTED) == syms


def test_status_strings(lib):
    assert lib.defcon_abi_version() == 2
    assert lib.defcon_status_string(0) == b"DEFCON_OK"
    assert lib.defcon_status_string(5) == b"DEFCON_ERR_LIMIT"


def _conv(**kw):
    from paper_conf_ipps_jayaweeralwrk24_b200._binding import defcon_conv_t
    d = dict(stride_h=1, stride_w=1, pad_h=1, pad_w=1, dil_h=1, dil_w=1, offset_groups=1, bound=0,
             offset_dtype=0)
    d.update(kw)
    return defcon_conv_t(**d)


FAKE = 0x7F0000000000   # 16-byte aligned fake device address; never dereferenced


def _fwd(lib, x=FAKE, N=2, H=8, W=8, Cin=64, off=FAKE, mask=FAKE, w=FAKE, b=FAKE, Cout=64, K=3,
         cv=None, dtype=1, sampler=0, fp32_mode=1, y=FAKE):
    cv = cv or _conv()
    V = ctypes.c_void_p
    return lib.defcon_dcn_forward(V(x), N, H, W, Cin, V(off), V(mask), V(w), V(b), Cout, K, K, cv,
                                  dtype, sampler, fp32_mode, V(y), None, 0, None, None)


@pytest.mark.parametrize("kw,status", [
    (dict(N=0), 1), (dict(H=-1), 1), (dict(Cout=0), 1),
    (dict(cv="g3"), 1),                   # G does not divide Cin
    (dict(cv="s0"), 1),                   # zero stride
    (dict(cv="tiny"), 1),                 # empty output grid (H=1, pad 0, K=3)
    (dict(dtype=7), 1), (dict(sampler=9), 1), (dict(fp32_mode=4), 1),
    (dict(x=0), 1), (dict(off=0), 1), (dict(y=0), 1),
    (dict(x=FAKE + 8), 3), (dict(mask=FAKE + 4), 3), (dict(w=FAKE + 2), 3),
    (dict(x=FAKE + 16), 3),               # tensor-core path: x is gathered in 32-byte vectors
    (dict(cv="g16_bf16"), 2),             # Cin/G = 4, not a multiple of 8 for bf16
    (dict(cv="neg_bound"), 1),            # bounded deformation P must be >= 0
    (dict(cv="bf16_offsets"), 1),         # offsets / mask: DEFCON_F32 or DEFCON_F16 only
])
def test_dcn_forward_validation(lib, kw, status):
    cvs = {"g3": _conv(offset_groups=3), "s0": _conv(stride_h=0), "neg_bound": _conv(bound=-1), "bf16_offsets": _conv(offset_dtype=1),
           "tiny": _conv(pad_h=0, pad_w=0), "g16_bf16": _conv(offset_groups=16)}
    if kw.get("cv") in cvs:
        name = kw.pop("cv")
        kw["cv"] = cvs[name]
        if name == "tiny":
            kw.update(H=1, W=1)
    assert _fwd(lib, **kw) == status
    assert lib.defcon_last_error_detail() != b""


def test_dcn_forward_limit(lib):
    # N*H*W*Cin >= 2^31 is rejected before launch
    assert _fwd(lib, N=4096, H=128, W=128, Cin=64) == 5


def test_offset_branch_validation(lib):
    V = ctypes.c_void_p
    args = [V(FAKE), 1, 8, 8, 16, 1, V(FAKE), V(FAKE), V(FAKE), V(FAKE), V(FAKE), 3]
    big = 1 << 30
    assert lib.defcon_offset_dw_conv(*args, _conv(), V(0), V(FAKE), V(FAKE), big, None) == 1  # offset NULL
    assert lib.defcon_offset_dw_conv(*args, _conv(), V(FAKE + 4), V(FAKE), V(FAKE), big, None) == 3
    assert lib.defcon_offset_dw_conv(*args, _conv(offset_groups=64), V(FAKE), V(FAKE), V(FAKE), big,
                                     None) == 5
    assert lib.defcon_offset_dw_conv(*args, _conv(), V(FAKE), V(FAKE), V(FAKE), 16, None) == 5  # ws
    bad = list(args)
    bad[1] = 0
    assert lib.defcon_offset_dw_conv(*bad, _conv(), V(FAKE), V(FAKE), V(FAKE), big, None) == 1
    out = ctypes.c_size_t(0)
    assert lib.defcon_offset_workspace_size(1, 8, 8, 16, 3, _conv(), ctypes.byref(out)) == 0
    # one-pass kernel: one packed parameter block per 32-channel chunk (W2 hi / lo image for
    # OC = 27 -> 32 rows, 2 x 32 x 128 B, + 352 dw / BN floats, 1 KB-aligned); without a device
    # (no TMA encoder) the two-pass t buffers: tf32 hi / lo planes + W2 planes padded to 256 rows
    assert out.value in ((2 * 32 * 128 + 352 * 4 + 1023) // 1024 * 1024, (2 * 8 * 8 * 16 + 2 * 256 * 16) * 4)


def test_dcn_forward_x_byte_limit(lib):
    """fp32 x of 2^30 elements (4 GiB) passes the element-count limit but not the samplers'
    32-bit byte offsets: LIMIT before any launch; the same shape in bf16 (2 GiB) is accepted by
    the size query."""
    out = ctypes.c_size_t(0)
    # N=1, H=W=1024, Cin=1024, Cout=16, K=1 (pad 0): x = 2^30 elements
    assert lib.defcon_dcn_workspace_size(1, 1024, 1024, 1024, 16, 1, 1, _conv(pad_h=0, pad_w=0), 0, 0, 0,
                                         ctypes.byref(out)) == 5
    assert lib.defcon_dcn_workspace_size(1, 1024, 1024, 1024, 16, 1, 1, _conv(pad_h=0, pad_w=0), 1, 0, 0,
                                         ctypes.byref(out)) == 0


def test_offset_prepack_validation(lib):
    """defcon_offset_packed_size / defcon_offset_pack_params / defcon_offset_dw_conv_packed reject
    bad arguments before any launch (include/defcon.h)."""
    V, sz = ctypes.c_void_p, ctypes.c_size_t(0)
    assert lib.defcon_offset_packed_size(256, 3, 1, 1, ctypes.byref(sz)) == 0
    # 8 chunks of 32 channels, one 1 KB-aligned block each (W2 hi / lo for 27 -> 32 rows + dw / BN)
    assert sz.value == 8 * ((2 * 32 * 128 + 352 * 4 + 1023) // 1024 * 1024)
    assert lib.defcon_offset_packed_size(12, 3, 1, 1, ctypes.byref(sz)) == 2            # C % 8
    assert lib.defcon_offset_packed_size(256, 3, 64, 1, ctypes.byref(sz)) == 5          # OC > 256
    assert lib.defcon_offset_packed_size(0, 3, 1, 1, ctypes.byref(sz)) == 1
    P = [V(FAKE)] * 4
    assert lib.defcon_offset_pack_params(256, 3, 1, 1, *P, V(FAKE), 16, None) == 5      # too small
    assert lib.defcon_offset_pack_params(256, 3, 1, 1, *P, V(FAKE + 4), 1 << 30, None) == 3
    assert lib.defcon_offset_pack_params(256, 3, 1, 1, V(0), *P[1:], V(FAKE), 1 << 30, None) == 1
    args = [V(FAKE), 1, 8, 8, 16, 1, V(FAKE), 1 << 30, V(FAKE), 3]
    assert lib.defcon_offset_dw_conv_packed(*args, _conv(), V(0), V(FAKE), None) == 1     # offset NULL
    assert lib.defcon_offset_dw_conv_packed(*args, _conv(), V(FAKE + 4), V(FAKE), None) == 3
    bad = list(args)
    bad[5] = 7
    assert lib.defcon_offset_dw_conv_packed(*bad, _conv(), V(FAKE), V(FAKE), None) == 1   # dtype


def test_workspace_size_and_layer_size(lib):
    out = ctypes.c_size_t(99)
    # bf16 tensor-core path: stream-K counters + fp32 partial tiles
    assert lib.defcon_dcn_workspace_size(2, 8, 8, 64, 64, 3, 3, _conv(), 1, 0, 1, ctypes.byref(out)) == 0
    assert out.value > 0
    # fp32 CUDA-core path needs none
    assert lib.defcon_dcn_workspace_size(2, 8, 8, 64, 64, 3, 3, _conv(), 0, 0, 1, ctypes.byref(out)) == 0
    assert out.value == 0
    # fp32 on the tensor cores (3xTF32): counters + partials (W's tf32 planes inside them)
    assert lib.defcon_dcn_workspace_size(2, 8, 8, 64, 64, 3, 3, _conv(), 0, 0, 0, ctypes.byref(out)) == 0
    assert out.value > 0
    # ... which needs Cin/G % 32 == 0 (one 128-byte fp32 row per k-iteration)
    assert lib.defcon_dcn_workspace_size(2, 8, 8, 48, 64, 3, 3, _conv(), 0, 0, 0, ctypes.byref(out)) == 2
    assert lib.defcon_layer_workspace_size(2, 8, 8, 64, 1, 64, 3, _conv(), 1, 0, 1, ctypes.byref(out)) == 0
    # x (2*8*8*64*2) + offsets + mask + y, each 256-aligned
    assert out.value >= 2 * 8 * 8 * 64 * 2 * 2 + 2 * 64 * 9 * 3 * 4
    assert lib.defcon_dcn_workspace_size(2, 8, 8, 64, 64, 3, 3, _conv(offset_groups=3), 1, 0, 1,
                                         ctypes.byref(out)) == 1
    # the host entry owns no texture plan: TEX / HYBRID are refused before anything is enqueued
    for sampler in (1, 2):
        assert lib.defcon_layer_workspace_size(2, 8, 8, 64, 1, 64, 3, _conv(), 1, sampler, 1,
                                               ctypes.byref(out)) == 2


def test_workspace_counters_at_a_shape_independent_offset(lib):
    """The stream-K counters follow a partial-tile region of one device-wide size, so the
    workspace sizes of two shapes differ only by their counter bytes (one zero-filled
    workspace serves both; include/defcon.h, defcon_dcn_forward)."""
    a, b = ctypes.c_size_t(0), ctypes.c_size_t(0)
    assert lib.defcon_dcn_workspace_size(1, 8, 8, 64, 256, 3, 3, _conv(), 1, 0, 1, ctypes.byref(a)) == 0
    assert lib.defcon_dcn_workspace_size(64, 35, 35, 64, 256, 3, 3, _conv(), 1, 0, 1, ctypes.byref(b)) == 0
    tiles_a = -(-1 * 8 * 8 // 128)
    tiles_b = -(-64 * 35 * 35 // 128)
    assert b.value - a.value == ((2 * (-(-tiles_b // 2)) * 4 + 255) // 256 - (2 * (-(-tiles_a // 2)) * 4 + 255) // 256) * 256


def test_binding_rejects_host_tensors():
    import torch
    import paper_conf_ipps_jayaweeralwrk24_b200 as d
    x = torch.zeros(1, 4, 4, 16)
    with pytest.raises(ValueError):
        d.defcon_dcn_forward(x, torch.zeros(1, 4, 4, 1, 9, 2), None, torch.zeros(16, 3, 3, 16))


def test_product_never_imports_oracle():
    """The product package must not import, link or call oracle/ (fail loudly instead)."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_jayaweeralwrk24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in src.lower(), f


def test_deform_columns_validation(lib):
    """defcon_deform_columns rejects bad arguments before any launch (no GPU needed)."""
    V = ctypes.c_void_p
    lib.defcon_deform_columns.restype = ctypes.c_int

    def call(x=FAKE, N=1, H=8, W=8, Cin=64, off=FAKE, mask=FAKE, K=3, cv=None, dtype=1, cols=FAKE):
        return lib.defcon_deform_columns(V(x), N, H, W, Cin, V(off), V(mask), K, K, cv or _conv(), dtype,
                                         V(cols), None)

    assert call(N=0) == 1
    assert call(x=0) == 1 and call(cols=0) == 1
    assert call(cv=_conv(offset_groups=3)) == 1          # G does not divide Cin
    assert call(cols=FAKE + 8) == 3                      # misaligned
    assert call(cols=FAKE + 16) == 3 and call(x=FAKE + 16) == 3   # 32-byte vectors: 32-byte alignment
    assert call(cv=_conv(offset_groups=8)) == 2          # Cin/G = 8: 32-byte bf16 pieces need 16
    assert call(dtype=5) == 1

"""Pins for the fp64 oracle, run on CPU (-m "not gpu").

Each test checks the oracle against something other than itself: a closed form,
a hand-computed value (tests/golden), or an independent library routine
(torch.nn.functional.conv2d / grid_sample, torchvision.ops.deform_conv2d), in fp64.
Each is chosen so that a plausible slip in the oracle (dropped tap, swapped dy/dx,
transposed (i,j), wrong group index, off-by-one border, truncation instead of floor,
mask applied to the wrong tap) fails at least one of them.
"""
import os

import numpy as np
import pytest
import torch
import torch.nn.functional as F

from defcon_workloads import configs, inputs

HERE = os.path.dirname(os.path.abspath(__file__))
rng = np.random.default_rng(12345)


def nchw(a):
    return torch.from_numpy(np.ascontiguousarray(a, np.float64)).permute(0, 3, 1, 2)


def oihw(w):
    return torch.from_numpy(np.ascontiguousarray(w, np.float64)).permute(0, 3, 1, 2)


def nhwc(t):
    return t.permute(0, 2, 3, 1).contiguous().numpy()


def rand_layer(N=2, H=7, W=9, Cin=8, Cout=5, K=3, G=1, stride=1, pad=1, dil=1, seed=0):
    r = np.random.default_rng(seed)
    Ho = configs.out_size(H, K, stride, pad, dil)
    Wo = configs.out_size(W, K, stride, pad, dil)
    x = r.standard_normal((N, H, W, Cin))
    w = r.standard_normal((Cout, K, K, Cin))
    b = r.standard_normal(Cout)
    off = 1.5 * r.standard_normal((N, Ho, Wo, G, K * K, 2))
    m = r.random((N, Ho, Wo, G, K * K))
    return x, w, b, off, m, Ho, Wo


# ---------------------------------------------------------------- P1: Eq.1 special case
@pytest.mark.parametrize("stride,H,W", [(1, 7, 9), (2, 9, 8), (2, 35, 35)])
@pytest.mark.parametrize("dil", [1, 2])
def test_p1_zero_offsets_equal_regular_conv(oracle_mod, stride, H, W, dil):
    """Zero offsets, m = 1: Eq.2 reduces to Eq.1 == F.conv2d in fp64."""
    x, w, b, _, _, Ho, Wo = rand_layer(H=H, W=W, stride=stride, dil=dil, pad=dil, Cin=6, Cout=4)
    off = np.zeros((x.shape[0], Ho, Wo, 1, 9, 2))
    y = oracle_mod.dcn_forward(x, off, w, b, stride=stride, pad=dil, dil=dil)
    ref = nhwc(F.conv2d(nchw(x), oihw(w), torch.from_numpy(b), stride=stride, padding=dil,
                        dilation=dil))
    assert y.shape == ref.shape
    np.testing.assert_allclose(y, ref, rtol=0, atol=1e-12)


# ---------------------------------------------------------------- P2: integer offsets
def _shift(xt, dy, dx):
    """x'(q) = x(q + (dy, dx)) with zeros outside (NCHW)."""
    N, C, H, W = xt.shape
    out = torch.zeros_like(xt)
    ys, yd = (slice(dy, H), slice(0, H - dy)) if dy >= 0 else (slice(0, H + dy), slice(-dy, H))
    xs, xd = (slice(dx, W), slice(0, W - dx)) if dx >= 0 else (slice(0, W + dx), slice(-dx, W))
    out[:, :, yd, xd] = xt[:, :, ys, xs]
    return out


def test_p2_integer_offsets_are_shifted_taps(oracle_mod):
    """Per-tap integer offsets (distinct dy != dx per tap) give exactly shifted taps:
    y = b + sum_k conv_k(shift(x, dy_k, dx_k)) with the single-tap kernel k.  A swapped
    dy/dx, transposed (i,j) or misplaced tap index changes the result."""
    x, w, b, _, _, Ho, Wo = rand_layer(H=8, W=10, Cin=4, Cout=3, seed=3)
    N = x.shape[0]
    taps = [(1, 0), (0, -2), (2, 1), (-1, 3), (0, 0), (-3, -1), (1, 2), (2, -2), (-2, 0)]
    off = np.zeros((N, Ho, Wo, 1, 9, 2))
    for k, (dy, dx) in enumerate(taps):
        off[..., 0, k, 0] = dy
        off[..., 0, k, 1] = dx
    y = oracle_mod.dcn_forward(x, off, w, b)
    P = 5   # shift on a zero-extended domain so that padding taps can land inside the image
    xt = F.pad(nchw(x), (P, P, P, P))
    H, W = x.shape[1:3]
    ref = torch.zeros(N, 3, Ho, Wo, dtype=torch.float64) + torch.from_numpy(b)[None, :, None, None]
    for k, (dy, dx) in enumerate(taps):
        wk = torch.zeros(3, 4, 3, 3, dtype=torch.float64)
        i, j = divmod(k, 3)
        wk[:, :, i, j] = oihw(w)[:, :, i, j]
        xs = _shift(xt, dy, dx)[:, :, P - 1:P + H + 1, P - 1:P + W + 1]
        ref += F.conv2d(xs, wk)
    np.testing.assert_allclose(y, nhwc(ref), rtol=0, atol=1e-12)


# ---------------------------------------------------------------- P3: half-pixel closed form
def test_p3_half_pixel_equals_box_average(oracle_mod):
    """dp = (0.5, 0.5) on every tap: x(q + 0.5) is the mean of the 2x2 block at q
    (zeros outside), so y = conv2d of the 2x2 box average (avg_pool2d) of padded x."""
    x, w, b, _, _, Ho, Wo = rand_layer(H=7, W=6, Cin=3, Cout=2, seed=4)
    off = np.full((x.shape[0], Ho, Wo, 1, 9, 2), 0.5)
    y = oracle_mod.dcn_forward(x, off, w, b)
    xp = F.pad(nchw(x), (2, 2, 2, 2))
    xa = F.avg_pool2d(xp, 2, stride=1)        # xa[t] = x~(t - 2 + 0.5)
    # y(ho) = sum_i w_i x~(ho - 1 + i + 0.5) = sum_i w_i xa[ho + i + 1]
    ref = F.conv2d(xa[:, :, 1:, 1:], oihw(w), torch.from_numpy(b))
    ref = ref[:, :, :Ho, :Wo]
    np.testing.assert_allclose(y, nhwc(ref), rtol=0, atol=1e-12)


# ---------------------------------------------------------------- P4: far out of bounds
def test_p4_far_oob_gives_bias(oracle_mod):
    x, w, b, _, m, Ho, Wo = rand_layer(H=6, W=5, seed=5)
    s = np.where(rng.random((x.shape[0], Ho, Wo, 1, 9, 2)) < 0.5, -1, 1)
    off = s * (max(6, 5) + 1 + rng.random(s.shape) * 3)
    y = oracle_mod.dcn_forward(x, off, w, b, mask=m)
    assert np.array_equal(y, np.broadcast_to(b, y.shape))


# ---------------------------------------------------------------- P5: mask
def test_p5_mask_one_zero_linear(oracle_mod):
    x, w, b, off, m, Ho, Wo = rand_layer(seed=6, G=2)
    v1 = oracle_mod.dcn_forward(x, off, w, b, G=2)
    ones = oracle_mod.dcn_forward(x, off, w, b, mask=np.ones_like(m), G=2)
    assert np.array_equal(v1, ones)
    zeros = oracle_mod.dcn_forward(x, off, w, b, mask=np.zeros_like(m), G=2)
    assert np.array_equal(zeros, np.broadcast_to(b, zeros.shape))
    m2 = rng.random(m.shape)
    ya = oracle_mod.dcn_forward(x, off, w, b, mask=m, G=2) - b
    yb = oracle_mod.dcn_forward(x, off, w, b, mask=m2, G=2) - b
    yab = oracle_mod.dcn_forward(x, off, w, b, mask=m + 0.5 * m2, G=2) - b
    np.testing.assert_allclose(yab, ya + 0.5 * yb, rtol=0, atol=1e-11)


def test_p5_mask_is_per_tap(oracle_mod):
    """Masking only tap k equals the single-tap conv for that tap (k = i*Kw + j)."""
    x, w, b, _, _, Ho, Wo = rand_layer(H=6, W=7, Cin=3, Cout=2, seed=7)
    N = x.shape[0]
    off = np.zeros((N, Ho, Wo, 1, 9, 2))
    for k in range(9):
        m = np.zeros((N, Ho, Wo, 1, 9))
        m[..., 0, k] = 1.0
        y = oracle_mod.dcn_forward(x, off, w, b, mask=m)
        wk = torch.zeros(2, 3, 3, 3, dtype=torch.float64)
        i, j = divmod(k, 3)
        wk[:, :, i, j] = oihw(w)[:, :, i, j]
        ref = F.conv2d(nchw(x), wk, torch.from_numpy(b), padding=1)
        np.testing.assert_allclose(y, nhwc(ref), rtol=0, atol=1e-12)


# ---------------------------------------------------------------- P6: hand values
def test_p6_hand_computed_bilinear(oracle_mod):
    rows = np.loadtxt(os.path.join(HERE, "golden", "bilinear_2x2.txt"), comments="#")
    x = np.array([[1.0, 2.0], [3.0, 4.0]]).reshape(1, 2, 2, 1)
    w = np.ones((1, 1, 1, 1))
    for dy, dx, expect in rows:
        off = np.zeros((1, 2, 2, 1, 1, 2))
        off[..., 0] = dy
        off[..., 1] = dx
        y = oracle_mod.dcn_forward(x, off, w, None, pad=0)
        assert abs(y[0, 0, 0, 0] - expect) < 1e-12, (dy, dx, y[0, 0, 0, 0], expect)
        assert abs(oracle_mod.bilinear(x[0, :, :, 0], dy, dx) - expect) < 1e-12


# ---------------------------------------------------------------- P7: library routine
def test_p7_k1_equals_grid_sample(oracle_mod):
    """K=1 DCN == grid_sample(bilinear, zeros, align_corners=True) then a 1x1 conv."""
    N, H, W, C, Co = 2, 9, 11, 5, 4
    r = np.random.default_rng(8)
    x = r.standard_normal((N, H, W, C))
    w = r.standard_normal((Co, 1, 1, C))
    b = r.standard_normal(Co)
    off = 3.0 * r.standard_normal((N, H, W, 1, 1, 2))
    y = oracle_mod.dcn_forward(x, off, w, b, pad=0)
    py = np.arange(H)[None, :, None] + off[..., 0, 0, 0]
    px = np.arange(W)[None, None, :] + off[..., 0, 0, 1]
    grid = np.stack([2 * px / (W - 1) - 1, 2 * py / (H - 1) - 1], axis=-1)
    s = F.grid_sample(nchw(x), torch.from_numpy(grid), mode="bilinear", padding_mode="zeros",
                      align_corners=True)
    ref = F.conv2d(s, oihw(w), torch.from_numpy(b))
    np.testing.assert_allclose(y, nhwc(ref), rtol=0, atol=1e-12)


# ---------------------------------------------------------------- P8: groups
def test_p8_groups_sum_of_blocks(oracle_mod):
    """A G-group DCN equals the sum of per-block G=1 DCNs (R5: contiguous blocks)."""
    G, Cin = 4, 8
    x, w, b, off, m, Ho, Wo = rand_layer(Cin=Cin, G=G, seed=9)
    y = oracle_mod.dcn_forward(x, off, w, b, mask=m, G=G)
    Cg = Cin // G
    acc = np.broadcast_to(b, y.shape).copy()
    for g in range(G):
        sl = slice(g * Cg, (g + 1) * Cg)
        acc += oracle_mod.dcn_forward(x[..., sl], off[:, :, :, g:g + 1], w[..., sl], None,
                                      mask=m[:, :, :, g:g + 1])
    np.testing.assert_allclose(y, acc, rtol=0, atol=1e-11)


# ---------------------------------------------------------------- P9: torchvision
@pytest.mark.parametrize("G,stride,dil,mod", [(1, 1, 1, True), (2, 2, 1, True), (4, 1, 2, False),
                                               (1, 2, 2, True)])
def test_p9_matches_torchvision(oracle_mod, G, stride, dil, mod):
    tv = pytest.importorskip("torchvision.ops")
    x, w, b, off, m, Ho, Wo = rand_layer(N=2, H=11, W=9, Cin=8, Cout=6, G=G, stride=stride,
                                         dil=dil, pad=dil, seed=10 + G)
    off = off * 2.0
    y = oracle_mod.dcn_forward(x, off, w, b, mask=m if mod else None, stride=stride, pad=dil,
                               dil=dil, G=G)
    N = x.shape[0]
    off_t = torch.from_numpy(off.reshape(N, Ho, Wo, G * 9 * 2)).permute(0, 3, 1, 2)
    m_t = torch.from_numpy(m.reshape(N, Ho, Wo, G * 9)).permute(0, 3, 1, 2) if mod else None
    ref = tv.deform_conv2d(nchw(x), off_t, oihw(w), torch.from_numpy(b), stride=stride,
                           padding=dil, dilation=dil, mask=m_t)
    np.testing.assert_allclose(y, nhwc(ref), rtol=0, atol=1e-10)


def test_pixels_equals_grid(oracle_mod):
    x, w, b, off, m, Ho, Wo = rand_layer(seed=20, G=2)
    y = oracle_mod.dcn_forward(x, off, w, b, mask=m, G=2)
    idx = np.array([0, 5, 17, x.shape[0] * Ho * Wo - 1])
    yp = oracle_mod.dcn_pixels(x, off, w, idx, b, mask=m, G=2)
    assert np.array_equal(yp, y.reshape(-1, y.shape[-1])[idx])


# ---------------------------------------------------------------- P10: offset branch
@pytest.mark.parametrize("G,with_mask,stride,pad,dil", [
    (1, True, 1, 1, 1), (4, True, 2, 1, 1), (2, False, 1, 1, 1),
    # geometry other than pad = dil = 1 (R10: the branch uses the DCN's stride/pad/dil)
    (1, True, 1, 2, 2), (1, True, 2, 0, 1), (2, True, 2, 3, 3), (1, False, 1, 0, 2)])
def test_p10_offset_branch_matches_torch(oracle_mod, G, with_mask, stride, pad, dil):
    r = np.random.default_rng(30 + G + 7 * pad + 13 * dil)
    N, H, W, C, K = 2, 9, 8, 6, 3
    x = r.standard_normal((N, H, W, C))
    dw = r.standard_normal((C, 3, 3))
    sc, sh = r.uniform(0.5, 1.5, C), 0.3 * r.standard_normal(C)
    OC = G * K * K * (3 if with_mask else 2)
    w2, b2 = r.standard_normal((OC, C)), r.standard_normal(OC)
    off, msk = oracle_mod.offset_branch(x, dw, sc, sh, w2, b2, K=K, G=G, with_mask=with_mask,
                                        stride=stride, pad=pad, dil=dil)
    t = F.conv2d(nchw(x), torch.from_numpy(dw)[:, None], stride=stride, padding=pad, dilation=dil,
                 groups=C)
    t = torch.relu(t * torch.from_numpy(sc)[None, :, None, None]
                   + torch.from_numpy(sh)[None, :, None, None])
    u = F.conv2d(t, torch.from_numpy(w2)[:, :, None, None], torch.from_numpy(b2))
    u = nhwc(u)
    n_off = 2 * G * K * K
    np.testing.assert_allclose(off.reshape(*off.shape[:3], -1), u[..., :n_off], rtol=0, atol=1e-12)
    if with_mask:
        np.testing.assert_allclose(msk.reshape(*msk.shape[:3], -1),
                                   torch.sigmoid(torch.from_numpy(u[..., n_off:])).numpy(),
                                   rtol=0, atol=1e-14)
    else:
        assert msk is None


def test_p10_zero_w2_gives_bias(oracle_mod):
    r = np.random.default_rng(40)
    x = r.standard_normal((1, 5, 5, 4))
    OC = 27
    b2 = r.standard_normal(OC)
    off, msk = oracle_mod.offset_branch(x, r.standard_normal((4, 3, 3)), np.ones(4), np.zeros(4),
                                        np.zeros((OC, 4)), b2)
    assert np.array_equal(off[0, 2, 3].reshape(-1), b2[:18])
    np.testing.assert_allclose(msk[0, 1, 1].reshape(-1), 1 / (1 + np.exp(-b2[18:])), atol=1e-15)


# ---------------------------------------------------------------- P11: continuity
def test_p11_continuity(oracle_mod):
    """Eq.3 is continuous: crossing an integer grid line changes y by O(eps)."""
    x, w, b, off, m, Ho, Wo = rand_layer(seed=50)
    off = np.round(off)
    ya = oracle_mod.dcn_forward(x, off - 1e-9, w, b, mask=m)
    yb = oracle_mod.dcn_forward(x, off + 1e-9, w, b, mask=m)
    assert np.max(np.abs(ya - yb)) < 1e-6


# ---------------------------------------------------------------- P13: texture model
def test_p13_texq_exact_on_256th_grid(oracle_mod):
    """With fractions already multiples of 1/256 the quantised filter is exact."""
    x, w, b, off, m, Ho, Wo = rand_layer(seed=60)
    off = np.round(off * 256) / 256
    ye = oracle_mod.dcn_forward(x, off, w, b, mask=m)
    for q in ("round", "trunc"):
        yq = oracle_mod.dcn_forward_texq(x, off, w, b, mask=m, quant=q)
        np.testing.assert_allclose(yq, ye, rtol=0, atol=1e-12)


def test_p13_texq_error_bound(oracle_mod):
    """Per-sample |quantised - exact| <= (|da_y| + |da_x|) * 2 max|x| with |da| <= 1/512
    (round) or < 1/256 (trunc); checked with K=1, w=1 so y is a single sample."""
    r = np.random.default_rng(61)
    x = r.standard_normal((1, 8, 8, 1))
    off = 3 * r.standard_normal((1, 8, 8, 1, 1, 2))
    w = np.ones((1, 1, 1, 1))
    ye = oracle_mod.dcn_forward(x, off, w, None, pad=0)
    for q, da in (("round", 1 / 512), ("trunc", 1 / 256)):
        yq = oracle_mod.dcn_forward_texq(x, off, w, None, pad=0, quant=q)
        bound = 2 * da * 2 * np.max(np.abs(x)) + 1e-12
        assert np.max(np.abs(yq - ye)) <= bound
        assert np.max(np.abs(yq - ye)) > 0


def test_p13_texq_closed_form(oracle_mod):
    """Texture model on the 2x2 image [[1,2],[3,4]] (f = 1 + x + 2y inside, K=1, w=1): the
    sample at (y, x) = (dy, dx) equals 1 + q(dx) + 2 q(dy), q the fraction quantised to 1/256
    (round: nearest 1/256; trunc: floor) -- the R14 model written out by hand."""
    x = np.array([1.0, 2.0, 3.0, 4.0]).reshape(1, 2, 2, 1)
    w = np.ones((1, 1, 1, 1))
    r = np.random.default_rng(62)
    f = r.uniform(0, 1, (1, 2, 2, 1, 1, 2))
    # every sample stays inside [0,1]^2: position (ho + dy, wo + dx) with the integer part removed
    pos = np.stack(np.meshgrid(np.arange(2), np.arange(2), indexing="ij"), -1).reshape(1, 2, 2, 1, 1, 2)
    off = f - pos
    for q, fn in (("round", lambda v: np.floor(v * 256 + 0.5) / 256), ("trunc", lambda v: np.floor(v * 256) / 256)):
        yq = oracle_mod.dcn_forward_texq(x, off, w, None, pad=0, quant=q)[..., 0]
        expect = 1 + fn(f[..., 1]) + 2 * fn(f[..., 0])
        np.testing.assert_allclose(yq, expect.reshape(1, 2, 2), rtol=0, atol=1e-14)


def test_p13_texq_hw_hand_value(oracle_mod):
    """The measured half4 filter model ("hw", R14), worked by hand with K = 1, w = 1.
    (a) [[1,2],[3,4]] at (dy, dx) = (0.7, 0.3): a = rne(76.8)/256 = 77/256, b = rne(179.2)/256
        = 179/256; weights*256 = rne(179*77/256 = 53.84) = 54, rne(77*77/256 = 23.16) = 23,
        rne(179*179/256 = 125.16) = 125, rne(77*179/256) = 54;
        value = (54*1 + 23*2 + 125*3 + 54*4)/256 = 691/256 (binary16-exact).
    (b) [[0,0],[0,1]] at (0.21, 0.37): value = w11 = ab; a = rne(94.72) = 95, b = rne(53.76)
        = 54 (in 1/256), w11 = rne(95*54/256 = 20.04)/256 = 20/256, while the fraction-only
        model ("round") keeps the unrounded product 95*54/65536."""
    w = np.ones((1, 1, 1, 1))
    pad_ = ((0, 0), (0, 1), (0, 1), (0, 0), (0, 0), (0, 0))   # 2x2 output grid, sample (0, 0)
    x = np.array([1.0, 2.0, 3.0, 4.0]).reshape(1, 2, 2, 1)
    off = np.pad(np.array([0.7, 0.3]).reshape(1, 1, 1, 1, 1, 2), pad_)
    assert oracle_mod.dcn_forward_texq(x, off, w, None, pad=0, quant="hw")[0, 0, 0, 0] == 691 / 256
    xs = np.array([0.0, 0.0, 0.0, 1.0]).reshape(1, 2, 2, 1)
    off = np.pad(np.array([0.21, 0.37]).reshape(1, 1, 1, 1, 1, 2), pad_)
    assert oracle_mod.dcn_forward_texq(xs, off, w, None, pad=0, quant="hw")[0, 0, 0, 0] == 20 / 256
    yr = oracle_mod.dcn_forward_texq(xs, off, w, None, pad=0, quant="round")[0, 0, 0, 0]
    assert abs(yr - 95 * 54 / 65536) < 1e-15


def test_p13_texq_hw_exact_cases_and_bound(oracle_mod):
    """"hw" model: with fractions on the 1/16 grid every weight product is a multiple of 1/256
    and small-integer texels keep the sum binary16-exact, so it equals the exact oracle; in
    general it stays within fraction rounding (2 x 1/512 x 2 max|x|) + weight rounding
    (4 x 1/512 max|x|) + binary16 rounding (2^-11 max|x|) of it (K = 1, w = 1)."""
    r = np.random.default_rng(64)
    x = r.integers(-8, 9, (1, 8, 8, 1)).astype(np.float64)
    off = np.round(3 * r.standard_normal((1, 8, 8, 1, 1, 2)) * 16) / 16
    w = np.ones((1, 1, 1, 1))
    ye = oracle_mod.dcn_forward(x, off, w, None, pad=0)
    yh = oracle_mod.dcn_forward_texq(x, off, w, None, pad=0, quant="hw")
    assert np.array_equal(ye, yh)
    x = r.standard_normal((1, 8, 8, 1))
    off = 3 * r.standard_normal((1, 8, 8, 1, 1, 2))
    ye = oracle_mod.dcn_forward(x, off, w, None, pad=0)
    yh = oracle_mod.dcn_forward_texq(x, off, w, None, pad=0, quant="hw")
    mx = np.max(np.abs(x))
    assert np.max(np.abs(yh - ye)) <= (4 / 512 + 4 / 512 + 2.0 ** -11) * mx
    assert np.max(np.abs(yh - ye)) > 0


def test_p13_texq_pixels_equals_grid(oracle_mod):
    x, w, b, off, m, Ho, Wo = rand_layer(seed=63, G=2)
    idx = np.array([0, 3, 11, x.shape[0] * Ho * Wo - 1])
    for q in ("round", "trunc", "hw"):
        y = oracle_mod.dcn_forward_texq(x, off, w, b, mask=m, G=2, quant=q)
        yp = oracle_mod.dcn_pixels(x, off, w, idx, b, mask=m, G=2, quant=q)
        assert np.array_equal(yp, y.reshape(-1, y.shape[-1])[idx])


# ---------------------------------------------------------------- P14: FLOP model
def test_p14_eq9_mac_saving():
    """Eq.9 prints 83.3% for k = 3."""
    assert round(100 * configs.lightweight_mac_saving(3), 1) == 83.3
    c = configs.C4.replace(modulated=False)
    regular = c.M * c.Cin * 9 * 2 * 9
    assert abs(1 - configs.offset_branch_macs(c) / regular - 0.8333333) < 1e-6


def test_flop_model_values():
    """11.23 / 23.12 / 48.92 GFLOP for C3 / C4 / C5."""
    for c, gf in ((configs.C3, 11.23), (configs.C4, 23.12), (configs.C5, 48.92)):
        assert round(configs.contraction_flops(c) / 1e9, 2) == gf
    assert len(configs.stack_layers()) == 11


def test_out_size_matches(oracle_mod):
    for args in [(35, 3, 2, 1, 1), (69, 3, 1, 1, 1), (2, 3, 2, 0, 1), (1, 3, 1, 0, 1), (18, 3, 1, 1, 2)]:
        assert oracle_mod.out_size(*args) == configs.out_size(*args)


def test_inputs_are_seeded_per_image():
    c = configs.C4.replace(N=3, H=5, W=5, Cin=8, Cout=8)
    full = inputs.gen_x(c)
    part = inputs.gen_x(c, images=[2])
    assert np.array_equal(full[2:3], part)
    xb = inputs.gen_x(c)
    assert np.array_equal(inputs.round_to(xb, "bf16"), xb)


# ------------------------------------------------------------------ deformable columns
def test_columns_zero_offsets_equal_unfold(oracle_mod):
    """Sampling step alone: zero offsets, no mask -> the regular im2col rows,
    i.e. F.unfold of the zero-padded input (fp64), reordered to [pixel][tap][ci]."""
    for stride, dil in ((1, 1), (2, 1), (1, 2)):
        x, _, _, off, _, _, _ = rand_layer(N=2, H=7, W=9, Cin=6, stride=stride, pad=dil, dil=dil, seed=3)
        off = np.zeros_like(off)
        cols = oracle_mod.deform_columns(x, off, 3, stride=stride, pad=dil, dil=dil)
        u = F.unfold(nchw(x), 3, dilation=dil, padding=dil, stride=stride)   # [N, Cin*9, L]
        N, Cin = x.shape[0], x.shape[3]
        ref = u.reshape(N, Cin, 9, -1).permute(0, 3, 2, 1).reshape(-1, 9 * Cin).numpy()
        assert cols.shape == ref.shape
        assert np.max(np.abs(cols - ref)) < 1e-14


def test_columns_times_weight_is_dcn(oracle_mod):
    """cols . W^T + b reproduces the (independently pinned) DCN forward, with mask and
    offset groups -- the columns carry every sampled, modulated value of Eq.2."""
    x, w, b, off, m, _, _ = rand_layer(N=2, H=6, W=8, Cin=8, Cout=5, G=2, seed=4)
    y = oracle_mod.dcn_forward(x, off, w, b, mask=m, G=2)
    idx = np.array([0, 5, 17, 33, 47, 95])
    cols = oracle_mod.deform_columns(x, off, 3, pix_idx=idx, mask=m, G=2)
    yy = cols @ w.reshape(w.shape[0], -1).T + b
    assert np.max(np.abs(yy - y.reshape(-1, w.shape[0])[idx])) < 1e-12


# ---------------------------------------------------------------- P15: bounded deformation
# P:182 (section III-A-c) restricts the learned offsets before the deformable kernel; reading
# R12: the sampling point of every tap is kept in the P x P window centred on the output
# pixel's centre tap (P = 7, Fig. 5).
def _off1(taps, K=3, G=1):
    """One pixel's offsets [1, 1, 1, G, K*K, 2] with the given {tap: (dy, dx)} set."""
    o = np.zeros((1, 1, 1, G, K * K, 2))
    for k, d in taps.items():
        o[0, 0, 0, 0, k] = d
    return o


@pytest.mark.parametrize("K,dil,P,tap,d,want", [
    # hand-worked: tap (i, j) sits r = ((i-1)d, (j-1)d) from the centre tap; h = (P-1)/2
    (3, 1, 7, 0, (-5.0, 2.5), (-2.0, 2.5)),     # r=(-1,-1): -6 -> -3 ; 1.5 inside
    (3, 1, 7, 7, (2.5, -4.0), (2.0, -3.0)),     # r=(1,0): 3.5 -> 3 ; -4 -> -3
    (3, 1, 7, 4, (0.25, 7.5), (0.25, 3.0)),     # centre tap: 7.5 -> 3
    (3, 2, 7, 2, (-1.5, 0.5), (-1.0, 0.5)),     # dil 2, r=(-2, 2): -3.5 -> -3 ; 2.5 inside
    (3, 1, 3, 0, (-0.5, 0.0), (0.0, 0.0)),      # P=3 (h=1), r=(-1,-1): -1.5 -> -1 ; -1 on the edge
    (2, 1, 2, 0, (-1.0, 0.2), (0.0, 0.2)),      # even K: r=(-0.5,-0.5), h=0.5: -1.5 -> -0.5
    (5, 1, 7, 24, (1.5, -9.0), (1.0, -5.0)),    # K=5, r=(2,2): 3.5 -> 3 ; -7 -> -3
])
def test_p15_bound_hand_values(oracle_mod, K, dil, P, tap, d, want):
    out = oracle_mod.bound_offsets(_off1({tap: d}, K=K), P, K=K, dil=dil)
    assert tuple(out[0, 0, 0, 0, tap]) == want


def test_p15_unbounded_and_inside_are_identity(oracle_mod):
    r = np.random.default_rng(15)
    off = r.uniform(-9, 9, (2, 3, 4, 2, 9, 2))
    assert np.array_equal(oracle_mod.bound_offsets(off, 0), off)          # P <= 0: unbounded
    inside = r.uniform(-2, 2, (2, 3, 4, 2, 9, 2))                          # |r + d| <= 3 for K=3
    assert np.array_equal(oracle_mod.bound_offsets(inside, 7), inside)
    b = oracle_mod.bound_offsets(off, 7)
    assert np.array_equal(oracle_mod.bound_offsets(b, 7), b)               # idempotent
    assert np.isnan(oracle_mod.bound_offsets(np.full((1, 1, 9, 2), np.nan), 7)).all()


@pytest.mark.parametrize("sign", [1, -1])
def test_p15_far_offsets_sample_the_window_corner(oracle_mod, sign):
    """Offsets of +-100 on every tap: bounded, every tap samples the window corner
    (centre + sign*3, centre + sign*3) exactly, so y = b + sum_k sum_c W[o,k,c] m_k x[corner, c]
    (0 outside the image) -- a closed form independent of the oracle's sampler."""
    x, w, b, _, m, Ho, Wo = rand_layer(H=9, W=8, Cin=4, Cout=3, seed=15)
    off = np.full((x.shape[0], Ho, Wo, 1, 9, 2), 100.0 * sign)
    y = oracle_mod.dcn_forward(x, oracle_mod.bound_offsets(off, 7), w, b, mask=m)
    ref = np.empty_like(y)
    N, H, W, _ = x.shape
    for n in range(N):
        for ho in range(Ho):
            for wo in range(Wo):
                yy, xx = ho + 3 * sign, wo + 3 * sign         # centre tap (ho, wo) with pad 1
                v = x[n, yy, xx] if (0 <= yy < H and 0 <= xx < W) else np.zeros(x.shape[3])
                wm = np.einsum("okc,k->oc", w.reshape(w.shape[0], 9, -1), m[n, ho, wo, 0])
                ref[n, ho, wo] = b + wm @ v
    np.testing.assert_allclose(y, ref, rtol=0, atol=1e-12)


# ---------------------------------------------------------------- P16: tex2D++ 16-bit offsets
# tex2D++ "only use[s] 16 bits to compute the offset"; reading R13: IEEE binary16 with
# round-to-nearest-even storage of offsets and mask.  Pinned to numpy's float16 conversion (a
# library routine) over normal, subnormal, tie and overflow values.
def test_p16_round_f16_matches_numpy(oracle_mod):
    r = np.random.default_rng(16)
    v = np.concatenate([r.uniform(-8, 8, 4000), r.standard_normal(2000) * 1e-5,       # subnormal range
                        np.array([1 + 2.0 ** -11, 1 + 3 * 2.0 ** -11, 2049.0, 2051.0,  # ties -> even
                                  65504.0, 65520.0, -70000.0, 2.0 ** -25, 0.0, -0.0])])
    got = oracle_mod.round_f16(v)
    want = v.astype(np.float16).astype(np.float64)
    assert np.array_equal(got, want)


def test_p16_f16_offsets_dcn_is_dcn_of_rounded(oracle_mod):
    """The 16-bit-offset DCN is the plain DCN on the rounded offsets and mask: equal to the
    torchvision-pinned DCN at those inputs, and within the rounding's effect of the fp32 one."""
    x, w, b, off, m, Ho, Wo = rand_layer(seed=16)
    o16, m16 = oracle_mod.round_f16(off), oracle_mod.round_f16(m)
    assert np.all(np.abs(o16 - off) <= 2.0 ** -11 * np.abs(off) + 2.0 ** -25)
    y16 = oracle_mod.dcn_forward(x, o16, w, b, mask=m16)
    y = oracle_mod.dcn_forward(x, off, w, b, mask=m)
    assert 0 < np.max(np.abs(y16 - y)) < 1e-2 * np.max(np.abs(y))

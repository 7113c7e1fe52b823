"""Seeded synthetic inputs with the shapes and distributions of the paper's workloads.

Recipe:
  seed(config, tensor, image) = 1_000_003*config_id + 1009*tensor_id + image
  x        ReLU(N(0,1))  (post conv1/BN/ReLU activations of a bottleneck);
           "normal" = N(0,1) stress case.  bf16 configs are rounded to bf16 (RNE).
  offsets  N(0, 1.5^2) px ("normal"); U(-7,7) ("local", the P=7 window of P:182);
           special sets: zeros, integers in [-3,3], half (0.5), far-OOB +-(H+2),
           border (values in (-1,0)).
  mask     sigmoid(N(0,1)).
  weight   N(0, 2/(Cin K^2)) (bf16-rounded for bf16 configs); bias N(0, 0.01^2).
  offset branch: W1 ~ N(0, 1/9); folded-BN scale U(0.5,1.5), shift N(0, 0.1^2);
           W2 scaled so that the produced offsets have std ~ 1.5 px; b2 N(0, 0.1^2).
Every array is generated per image so any rank can regenerate exactly its shard.
No method arithmetic lives here: values are drawn, rounded to the storage dtype
and returned as numpy float32 arrays (exactly representable in the storage dtype).
"""
from __future__ import annotations

import numpy as np
import torch

from .configs import LayerConfig

T_X, T_OFF, T_MASK, T_W, T_B, T_W1, T_BNS, T_BNB, T_W2, T_B2 = range(10)


def seed_for(config_id: int, tensor_id: int, image: int = 0) -> int:
    return 1_000_003 * config_id + 1009 * tensor_id + image


def _rng(config_id, tensor_id, image=0):
    return np.random.default_rng(seed_for(config_id, tensor_id, image))


def round_to(a: np.ndarray, dtype: str) -> np.ndarray:
    """Round fp32 values to the storage dtype (bf16: round-to-nearest-even) and return fp32."""
    a = np.ascontiguousarray(a, dtype=np.float32)
    if dtype == "f32":
        return a
    if dtype == "bf16":
        return torch.from_numpy(a).to(torch.bfloat16).to(torch.float32).numpy()
    if dtype == "f16":
        return a.astype(np.float16).astype(np.float32)
    raise ValueError(dtype)


def gen_x(c: LayerConfig, images=None, dist: str = "relu") -> np.ndarray:
    images = range(c.N) if images is None else images
    out = []
    for n in images:
        v = _rng(c.config_id, T_X, n).standard_normal((c.H, c.W, c.Cin), dtype=np.float32)
        if dist == "relu":
            v = np.maximum(v, 0.0)
        out.append(v)
    return round_to(np.stack(out), c.dtype)


def gen_offsets(c: LayerConfig, images=None, dist: str = "normal") -> np.ndarray:
    images = range(c.N) if images is None else images
    KK = c.K * c.K
    shape = (c.Ho, c.Wo, c.G, KK, 2)
    out = []
    for n in images:
        r = _rng(c.config_id, T_OFF, n)
        if dist == "normal":
            v = 1.5 * r.standard_normal(shape, dtype=np.float32)
        elif dist == "local":
            v = r.uniform(-7.0, 7.0, shape).astype(np.float32)
        elif dist == "zeros":
            v = np.zeros(shape, np.float32)
        elif dist == "integer":
            v = r.integers(-3, 4, shape).astype(np.float32)
        elif dist == "half":
            v = np.full(shape, 0.5, np.float32)
        elif dist == "far":
            v = (np.where(r.random(shape) < 0.5, -1.0, 1.0) * (max(c.H, c.W) + 2)).astype(np.float32)
        elif dist == "border":
            v = -r.random(shape).astype(np.float32)       # in (-1, 0]
        else:
            raise ValueError(dist)
        out.append(v)
    return np.ascontiguousarray(np.stack(out), dtype=np.float32)


def gen_mask(c: LayerConfig, images=None) -> np.ndarray:
    images = range(c.N) if images is None else images
    KK = c.K * c.K
    out = []
    for n in images:
        z = _rng(c.config_id, T_MASK, n).standard_normal((c.Ho, c.Wo, c.G, KK), dtype=np.float32)
        out.append(1.0 / (1.0 + np.exp(-z)))
    return np.ascontiguousarray(np.stack(out), dtype=np.float32)


def gen_weight(c: LayerConfig):
    """weight [Cout, K, K, Cin] (storage-dtype rounded), bias [Cout] fp32."""
    KK = c.K * c.K
    w = _rng(c.config_id, T_W).standard_normal((c.Cout, c.K, c.K, c.Cin), dtype=np.float32)
    w = w * np.float32(np.sqrt(2.0 / (c.Cin * KK)))
    b = (0.01 * _rng(c.config_id, T_B).standard_normal(c.Cout)).astype(np.float32)
    return round_to(w, c.dtype), b


def gen_offset_branch(c: LayerConfig, target_std: float = 1.5):
    """Parameters of the lightweight offset branch, fp32.

    Returns dict(dw_w [C,3,3], dw_scale [C], dw_shift [C], pw_w [OC,C], pw_b [OC]).
    W2 rows for offsets are scaled so offsets have std ~ target_std px for ReLU(N(0,1))
    inputs; mask-logit rows get std ~ 1.
    """
    C = c.Cin
    KK = c.K * c.K
    n_off = 2 * c.G * KK
    OC = n_off + (c.G * KK if c.modulated else 0)
    dw_w = (_rng(c.config_id, T_W1).standard_normal((C, 3, 3)) / 3.0).astype(np.float32)
    dw_scale = _rng(c.config_id, T_BNS).uniform(0.5, 1.5, C).astype(np.float32)
    dw_shift = (0.1 * _rng(c.config_id, T_BNB).standard_normal(C)).astype(np.float32)
    # E[t^2] for t = ReLU(s*z + b), z ~ dw-conv of ReLU(N(0,1)) inputs: estimate the scale
    # of t analytically-ish: var(z) ~ 9 * (1/9) * E[x^2] = 0.5, so t has rms ~ 0.5 * s.
    t_rms = 0.5
    w2 = _rng(c.config_id, T_W2).standard_normal((OC, C)).astype(np.float32)
    w2[:n_off] *= np.float32(target_std / (t_rms * np.sqrt(C)))
    w2[n_off:] *= np.float32(1.0 / (t_rms * np.sqrt(C)))
    b2 = (0.1 * _rng(c.config_id, T_B2).standard_normal(OC)).astype(np.float32)
    return dict(dw_w=dw_w, dw_scale=dw_scale, dw_shift=dw_shift, pw_w=w2, pw_b=b2)


def gen_layer(c: LayerConfig, images=None, x_dist="relu", off_dist="normal"):
    """All DCN-stage inputs for one layer: dict(x, offset, mask|None, weight, bias)."""
    w, b = gen_weight(c)
    return dict(x=gen_x(c, images, x_dist), offset=gen_offsets(c, images, off_dist),
                mask=gen_mask(c, images) if c.modulated else None, weight=w, bias=b)

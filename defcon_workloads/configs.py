"""BASELINE.json configurations and the FLOP / byte model.

Shapes are the YOLACT++ ResNet-101 DCN layers at a 550x550 input (
stage sizes 138 -> 69 -> 35 -> 18, table after Fig.7).  All layers use
a 3x3 kernel, pad 1, dilation 1 (the bottleneck 3x3 conv).
"""
from __future__ import annotations

import dataclasses
from typing import List


@dataclasses.dataclass(frozen=True)
class LayerConfig:
    name: str
    N: int
    Cin: int
    Cout: int
    H: int
    W: int
    K: int = 3
    stride: int = 1
    pad: int = 1
    dil: int = 1
    G: int = 1               # offset (deformable) groups
    modulated: bool = True   # DCNv2 mask (R6)
    dtype: str = "bf16"      # "bf16" or "f32" (x, W, y)
    config_id: int = 0       # seeds (inputs.seed_for)

    @property
    def Ho(self) -> int:
        return out_size(self.H, self.K, self.stride, self.pad, self.dil)

    @property
    def Wo(self) -> int:
        return out_size(self.W, self.K, self.stride, self.pad, self.dil)

    @property
    def M(self) -> int:
        return self.N * self.Ho * self.Wo

    def replace(self, **kw) -> "LayerConfig":
        return dataclasses.replace(self, **kw)


def out_size(n_in: int, k: int, stride: int, pad: int, dil: int) -> int:
    """Regular-conv output extent ("computed similarly to a regular convolution")."""
    span = n_in + 2 * pad - dil * (k - 1) - 1
    return 0 if span < 0 else span // stride + 1


# BASELINE.json "configs", in order.
TINY = LayerConfig("tiny_v1_f32", N=1, Cin=16, Cout=16, H=16, W=16, G=1, modulated=False,
                   dtype="f32", config_id=1)
C3 = LayerConfig("yolact_r101_c3_v2", N=8, Cin=128, Cout=128, H=69, W=69, config_id=2)
C4 = LayerConfig("yolact_r101_c4_v2", N=16, Cin=256, Cout=256, H=35, W=35, config_id=3)
C4_G4 = C4.replace(name="yolact_r101_c4_v2_g4", G=4)
C4_F32 = C4.replace(name="yolact_r101_c4_v2_f32", dtype="f32")
C4_G4_F32 = C4.replace(name="yolact_r101_c4_v2_g4_f32", G=4, dtype="f32")
C5 = LayerConfig("yolact_r101_c5_v2", N=32, Cin=512, Cout=512, H=18, W=18, config_id=4)

SINGLE_LAYER = {c.name: c for c in (TINY, C3, C4, C4_G4, C4_F32, C4_G4_F32, C5)}


def stack_layers(batch: int = 64) -> List[LayerConfig]:
    """Config 5: YOLACT++ interval-3 placement over R101 C3-C5.

    Every 3rd bottleneck (i % 3 == 0) of C3 (4 blocks), C4 (23) and C5 (3) gets a
    DCN (11 layers).  Block 0 of each stage is the stride-2 one and
    sees the previous stage's spatial size.
    """
    layers = []
    stages = [("c3", 128, 138, 69, 4), ("c4", 256, 69, 35, 23), ("c5", 512, 35, 18, 3)]
    for sname, C, h_in, h_out, nblocks in stages:
        for b in range(0, nblocks, 3):
            if b == 0:
                layers.append(LayerConfig(f"stack_{sname}b{b}", N=batch, Cin=C, Cout=C, H=h_in,
                                          W=h_in, stride=2, config_id=5))
            else:
                layers.append(LayerConfig(f"stack_{sname}b{b}", N=batch, Cin=C, Cout=C, H=h_out,
                                          W=h_out, stride=1, config_id=5))
    return layers


# ---------------------------------------------------------------- FLOP / byte model
def contraction_flops(c: LayerConfig) -> int:
    """2 * M * Cout * K^2 * Cin: the dense contraction only."""
    return 2 * c.M * c.Cout * c.K * c.K * c.Cin


def elem_bytes(dtype: str) -> int:
    return {"bf16": 2, "f32": 4}[dtype]


def dcn_compulsory_bytes(c: LayerConfig) -> int:
    """x, offsets, mask, W, bias read once + y written once (fp32 offsets/mask/bias)."""
    e = elem_bytes(c.dtype)
    KK = c.K * c.K
    b = c.N * c.H * c.W * c.Cin * e                 # x
    b += c.M * c.G * KK * 2 * 4                      # offsets
    if c.modulated:
        b += c.M * c.G * KK * 4                      # mask
    b += c.Cout * KK * c.Cin * e                     # W
    b += c.Cout * 4                                  # bias
    b += c.M * c.Cout * e                            # y
    return b


def offset_branch_oc(c: LayerConfig) -> int:
    return c.G * c.K * c.K * (3 if c.modulated else 2)


def offset_branch_macs(c: LayerConfig) -> int:
    """dw 3x3 (9 C per output pixel) + 1x1 (C * OC per output pixel)."""
    return c.M * (9 * c.Cin + c.Cin * offset_branch_oc(c))


def offset_branch_compulsory_bytes(c: LayerConfig) -> int:
    e = elem_bytes(c.dtype)
    KK = c.K * c.K
    b = c.N * c.H * c.W * c.Cin * e                  # x read once
    b += c.Cin * (9 + 2) * 4 + offset_branch_oc(c) * (c.Cin + 1) * 4   # weights
    b += c.M * c.G * KK * 2 * 4                      # offsets written
    if c.modulated:
        b += c.M * c.G * KK * 4                      # mask written
    return b


def lightweight_mac_saving(k: int) -> float:
    """Eq.9: MACs saved by replacing the regular 3x3 offset conv (2k^2 x C x 3 x 3)
    with dw 3x3 (C x 1 x 3 x 3) + 1x1 (2k^2 x C).  H, W, C cancel."""
    regular = 3 * 3 * 2 * k * k
    light = 3 * 3 + 2 * k * k
    return 1.0 - light / regular

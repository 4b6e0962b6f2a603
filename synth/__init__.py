"""Seeded synthetic workloads shared by the tests, the bench and the oracle runs.

This module holds ONLY shapes and random-number recipes -- none of the
method's arithmetic -- so that both the CUDA path's tests and the oracle can
draw identical inputs without sharing any code with each other (DESIGN.md
§Inputs).  The paper uses random inputs because convolution performance is
value-independent (PAPER.md P.1415-1419, P.1458-1461).

Recipes:
  "uniform": x ~ U(-1,1); w ~ U(-1,1)/sqrt(C*R*S)  (outputs are O(1))
  "int":     x ~ integers in [-8,8], w ~ integers in [-4,4]  (every precision
             is exact: products/partial sums are integers < 2^24)
  "small":   x ~ integers in [-2,2], w ~ integers in [-2,2]
Seeds: numpy default_rng(20250301 + 1000*config_id + layer_id) unless given.
"""
from __future__ import annotations

from dataclasses import dataclass, asdict

import numpy as np

BASE_SEED = 20250301


@dataclass(frozen=True)
class ConvShape:
    name: str
    N: int
    C: int
    H: int
    W: int
    K: int
    R: int
    S: int
    sh: int = 1
    sw: int = 1
    ph: int = 0
    pw: int = 0
    count: int = 1          # how many times the shape occurs in its network

    @property
    def stride(self):
        return (self.sh, self.sw)

    @property
    def padding(self):
        return (self.ph, self.pw)

    @property
    def P(self):
        return (self.H + 2 * self.ph - self.R) // self.sh + 1

    @property
    def Q(self):
        return (self.W + 2 * self.pw - self.S) // self.sw + 1

    def flops(self) -> int:
        """Algorithmic FLOPs 2*N*K*C*R*S*P*Q (BASELINE.json north_star)."""
        return 2 * self.N * self.K * self.C * self.R * self.S * self.P * self.Q

    def bytes(self, eb_x: int, eb_w: int, eb_y: int) -> int:
        """Algorithmic bytes: unpacked x read once, w once, y written once
        (SURVEY §8(d))."""
        return (eb_x * self.N * self.C * self.H * self.W + eb_w * self.K * self.C * self.R * self.S
                + eb_y * self.N * self.K * self.P * self.Q)

    def with_batch(self, N: int) -> "ConvShape":
        d = asdict(self)
        d["N"] = N
        return ConvShape(**d)

    def asdict(self):
        return asdict(self)


def _same(name, N, C, K, H, R, s=1, count=1):
    """Torch-style 'same-ish' conv: pad R//2."""
    return ConvShape(name, N, C, H, H, K, R, R, s, s, R // 2, R // 2, count)


# BASELINE.json configs[0]: tiny CPU-oracle check
TINY = ConvShape("tiny", 1, 1, 8, 8, 1, 3, 3)

# configs[1]: ResNet-50 conv3_x layer
CONV3X = ConvShape("resnet50_conv3x", 32, 128, 28, 28, 128, 3, 3, 1, 1, 1, 1)

# configs[2]: VGG-16 13 conv layers, N=64, 3x3 s1 p1
VGG16 = [
    _same("conv1_1", 64, 3, 64, 224, 3), _same("conv1_2", 64, 64, 64, 224, 3),
    _same("conv2_1", 64, 64, 128, 112, 3), _same("conv2_2", 64, 128, 128, 112, 3),
    _same("conv3_1", 64, 128, 256, 56, 3), _same("conv3_2", 64, 256, 256, 56, 3),
    _same("conv3_3", 64, 256, 256, 56, 3), _same("conv4_1", 64, 256, 512, 28, 3),
    _same("conv4_2", 64, 512, 512, 28, 3), _same("conv4_3", 64, 512, 512, 28, 3),
    _same("conv5_1", 64, 512, 512, 14, 3), _same("conv5_2", 64, 512, 512, 14, 3),
    _same("conv5_3", 64, 512, 512, 14, 3),
]


def _sweep():
    pts = []
    for s in (1, 2):
        for h in (7, 14, 28, 56, 112, 224):          # A: Fig. 3 axis, 5x5 kernels
            pts.append(_same(f"A_h{h}_s{s}", 128, 64, 64, h, 5, s))
        for r in (1, 3, 5, 7):                        # B: Fig. 4 axis, kernel size
            pts.append(_same(f"B_r{r}_s{s}", 128, 64, 64, 56, r, s))
        for c in (16, 32, 64, 128, 256, 512):         # C: Fig. 5 axis, channels
            pts.append(_same(f"C_c{c}_s{s}", 32, c, c, 112, 3, s))
    pts.append(_same("D_c16_k512", 32, 16, 512, 56, 3))
    pts.append(_same("D_c512_k16", 32, 512, 16, 56, 3))
    return pts


# configs[3]: paper-style one-factor sweeps (34 points)
SWEEP = _sweep()

# configs[4]: ResNet-50 v1.5 forward convs, N=256 (23 unique shapes, 53 convs)
RESNET50 = [
    ConvShape("stem7x7", 256, 3, 224, 224, 64, 7, 7, 2, 2, 3, 3, 1),
    ConvShape("l1_1x1_64_64", 256, 64, 56, 56, 64, 1, 1, 1, 1, 0, 0, 1),
    ConvShape("l1_3x3_64", 256, 64, 56, 56, 64, 3, 3, 1, 1, 1, 1, 3),
    ConvShape("l1_1x1_64_256", 256, 64, 56, 56, 256, 1, 1, 1, 1, 0, 0, 4),
    ConvShape("l1_1x1_256_64", 256, 256, 56, 56, 64, 1, 1, 1, 1, 0, 0, 2),
    ConvShape("l2_1x1_256_128", 256, 256, 56, 56, 128, 1, 1, 1, 1, 0, 0, 1),
    ConvShape("l2_3x3_128_s2", 256, 128, 56, 56, 128, 3, 3, 2, 2, 1, 1, 1),
    ConvShape("l2_1x1_128_512", 256, 128, 28, 28, 512, 1, 1, 1, 1, 0, 0, 4),
    ConvShape("l2_down_256_512_s2", 256, 256, 56, 56, 512, 1, 1, 2, 2, 0, 0, 1),
    ConvShape("l2_1x1_512_128", 256, 512, 28, 28, 128, 1, 1, 1, 1, 0, 0, 3),
    ConvShape("l2_3x3_128", 256, 128, 28, 28, 128, 3, 3, 1, 1, 1, 1, 3),
    ConvShape("l3_1x1_512_256", 256, 512, 28, 28, 256, 1, 1, 1, 1, 0, 0, 1),
    ConvShape("l3_3x3_256_s2", 256, 256, 28, 28, 256, 3, 3, 2, 2, 1, 1, 1),
    ConvShape("l3_1x1_256_1024", 256, 256, 14, 14, 1024, 1, 1, 1, 1, 0, 0, 6),
    ConvShape("l3_down_512_1024_s2", 256, 512, 28, 28, 1024, 1, 1, 2, 2, 0, 0, 1),
    ConvShape("l3_1x1_1024_256", 256, 1024, 14, 14, 256, 1, 1, 1, 1, 0, 0, 5),
    ConvShape("l3_3x3_256", 256, 256, 14, 14, 256, 3, 3, 1, 1, 1, 1, 5),
    ConvShape("l4_1x1_1024_512", 256, 1024, 14, 14, 512, 1, 1, 1, 1, 0, 0, 1),
    ConvShape("l4_3x3_512_s2", 256, 512, 14, 14, 512, 3, 3, 2, 2, 1, 1, 1),
    ConvShape("l4_1x1_512_2048", 256, 512, 7, 7, 2048, 1, 1, 1, 1, 0, 0, 3),
    ConvShape("l4_down_1024_2048_s2", 256, 1024, 14, 14, 2048, 1, 1, 2, 2, 0, 0, 1),
    ConvShape("l4_1x1_2048_512", 256, 2048, 7, 7, 512, 1, 1, 1, 1, 0, 0, 2),
    ConvShape("l4_3x3_512", 256, 512, 7, 7, 512, 3, 3, 1, 1, 1, 1, 2),
]

CONFIGS = {
    0: ("tiny", [TINY]),
    1: ("resnet50_conv3x", [CONV3X]),
    2: ("vgg16_n64", VGG16),
    3: ("sweep", SWEEP),
    4: ("resnet50_n256", RESNET50),
}


def seed_for(config_id: int, layer_id: int = 0) -> int:
    return BASE_SEED + 1000 * config_id + layer_id


def make_inputs(shape: ConvShape, seed: int, mode: str = "uniform", batch=None):
    """Return float32 numpy (x[N][C][H][W], w[K][C][R][S]).
    batch: optional (start, stop) subset of images; the full tensor is drawn
    image by image so a subset equals the same images of the full draw."""
    rng = np.random.default_rng(seed)
    N, C, H, W, K, R, S = shape.N, shape.C, shape.H, shape.W, shape.K, shape.R, shape.S
    # filters first so they do not depend on the batch subset
    if mode == "uniform":
        w = (rng.uniform(-1.0, 1.0, (K, C, R, S)) / np.sqrt(C * R * S)).astype(np.float32)
    elif mode == "int":
        w = rng.integers(-4, 5, (K, C, R, S)).astype(np.float32)
    elif mode == "small":
        w = rng.integers(-2, 3, (K, C, R, S)).astype(np.float32)
    else:
        raise ValueError(mode)
    lo, hi = (0, N) if batch is None else batch
    xs = []
    for n in range(N):
        img_rng = np.random.default_rng([seed, n])
        if n < lo or n >= hi:
            continue
        if mode == "uniform":
            xs.append(img_rng.uniform(-1.0, 1.0, (C, H, W)).astype(np.float32))
        elif mode == "int":
            xs.append(img_rng.integers(-8, 9, (C, H, W)).astype(np.float32))
        else:
            xs.append(img_rng.integers(-2, 3, (C, H, W)).astype(np.float32))
    x = np.stack(xs) if xs else np.zeros((0, C, H, W), np.float32)
    return x, w

"""Seeded synthetic inputs shaped like the paper's datasets (Table I).

Input generation only: nothing here is part of SONG's arithmetic, and both the
CUDA path and the oracle consume these arrays.  The recipes are stated in
DESIGN.md §5; seeds: data s, queries s+1, graph s+2.
Queries are fresh draws from the same generator, never members of the base set.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field
from typing import Optional

import torch


@dataclass
class Config:
    name: str
    n: int
    dim: int
    metric: str            # "l2" | "ip" | "cosine"
    degree: int
    nq: int
    K: int
    seed: int
    kind: str               # generator recipe
    queue_len: int = 64     # default operating point for parity tests
    extra: dict = field(default_factory=dict)


CONFIGS = {
    # BASELINE.json configs[0]: the oracle finishes it in seconds
    "tiny": Config("tiny", 10_000, 32, "l2", 16, 100, 10, 0, "gauss", 64),
    # configs[1]: the metric's workload (QPS at recall@10 = 0.95)
    "sift1m": Config("sift1m", 1_000_000, 128, "l2", 32, 10_000, 10, 100, "sift"),
    "gist1m": Config("gist1m", 1_000_000, 960, "l2", 32, 1_000, 10, 200, "gist"),
    "glove200": Config("glove200", 1_183_514, 200, "ip", 32, 10_000, 10, 300, "glove"),
    "nytimes256": Config("nytimes256", 289_761, 256, "cosine", 32, 10_000, 10, 400, "nytimes"),
    # §VII / Fig. 14: MNIST8m and its 1M sample, searched top-1 through
    # 1-bit random-projection codes of h bits (extra["hash_bits"])
    "mnist1m": Config("mnist1m", 1_000_000, 784, "l2", 32, 10_000, 1, 600, "mnist",
                      extra={"hash_bits": 128}),
    "mnist8m": Config("mnist8m", 8_090_000, 784, "l2", 32, 10_000, 1, 600, "mnist",
                      extra={"hash_bits": 128}),
}


def _gen(seed: int, device) -> torch.Generator:
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    return g


def gauss(n: int, dim: int, seed: int, device="cpu") -> torch.Tensor:
    """iid N(0, 1) (the tiny config)."""
    return torch.randn(n, dim, generator=_gen(seed, device), device=device, dtype=torch.float32)


class SiftLike:
    """SIFT-shaped ("less skewed"): latent z in R^16 from 1024
    equal-weight Gaussian clusters; x = relu(W z + b + eps), scaled to mean
    norm ~512 and rounded to integers in [0, 255] (so every L2 partial sum is
    an integer < 2^24: exact in fp32 in any order — pin P8)."""

    LATENT = 16
    CLUSTERS = 1024

    def __init__(self, dim: int, seed: int, device="cpu"):
        g = _gen(seed * 7919 + 17, device)
        self.dim, self.device = dim, device
        self.centers = torch.randn(self.CLUSTERS, self.LATENT, generator=g, device=device) * 1.5
        self.W = torch.randn(dim, self.LATENT, generator=g, device=device) / math.sqrt(self.LATENT)
        self.b = torch.randn(dim, generator=g, device=device) * 0.3 - 0.2
        # a fixed scale chosen so the mean row norm is ~512 (checked in tests)
        self.scale = 46.5 * math.sqrt(128.0 / dim)

    def sample(self, m: int, seed: int) -> torch.Tensor:
        g = _gen(seed, self.device)
        out = torch.empty(m, self.dim, device=self.device)
        step = 1 << 18
        for s in range(0, m, step):
            k = min(step, m - s)
            c = torch.randint(0, self.CLUSTERS, (k,), generator=g, device=self.device)
            z = self.centers[c] + 0.6 * torch.randn(k, self.LATENT, generator=g, device=self.device)
            x = z @ self.W.T + self.b + 0.25 * torch.randn(k, self.dim, generator=g, device=self.device)
            out[s:s + k] = torch.clamp(torch.round(torch.relu(x) * self.scale), 0, 255)
        return out


class GistLike:
    """GIST-shaped: non-negative, strongly correlated dims (latent 32), values in
    [0, ~0.5], row norm ~1."""

    LATENT = 32

    def __init__(self, dim: int, seed: int, device="cpu"):
        g = _gen(seed * 7919 + 17, device)
        self.dim, self.device = dim, device
        self.centers = torch.randn(256, self.LATENT, generator=g, device=device)
        self.W = torch.randn(dim, self.LATENT, generator=g, device=device).abs() / math.sqrt(self.LATENT)

    def sample(self, m: int, seed: int) -> torch.Tensor:
        g = _gen(seed, self.device)
        out = torch.empty(m, self.dim, device=self.device)
        step = 1 << 16
        for s in range(0, m, step):
            k = min(step, m - s)
            c = torch.randint(0, 256, (k,), generator=g, device=self.device)
            z = torch.relu(self.centers[c] + 0.7 * torch.randn(k, self.LATENT, generator=g,
                                                               device=self.device))
            x = z @ self.W.T + 0.05 * torch.rand(k, self.dim, generator=g, device=self.device)
            x = x / x.norm(dim=1, keepdim=True).clamp_min(1e-6)
            out[s:s + k] = x.clamp(0, 0.5)
        return out


class ClusteredSkewed:
    """GloVe / NYTimes shaped ("heavily skewed and clustered"): Zipf(1.1)
    cluster sizes over anisotropic clusters.  GloVe: log-normal row norms
    (sigma 0.3), so IP != cosine.  NYTimes: sparse-ish non-negative TF-IDF-like
    values (cosine metric normalises them)."""

    def __init__(self, dim: int, seed: int, clusters: int, nonneg: bool, device="cpu"):
        g = _gen(seed * 7919 + 17, device)
        self.dim, self.device, self.nonneg, self.C = dim, device, nonneg, clusters
        self.centers = torch.randn(clusters, dim, generator=g, device=device)
        self.axes = torch.randn(clusters, dim, generator=g, device=device).abs() + 0.1
        w = 1.0 / torch.arange(1, clusters + 1, device=device, dtype=torch.float64) ** 1.1
        self.p = (w / w.sum()).float()

    def sample(self, m: int, seed: int) -> torch.Tensor:
        g = _gen(seed, self.device)
        out = torch.empty(m, self.dim, device=self.device)
        step = 1 << 16
        for s in range(0, m, step):
            k = min(step, m - s)
            c = torch.multinomial(self.p, k, replacement=True, generator=g)
            x = self.centers[c] + 0.6 * self.axes[c] * torch.randn(k, self.dim, generator=g,
                                                                  device=self.device)
            if self.nonneg:
                x = torch.relu(x - 0.8)  # ~ 75 % zeros
            else:
                nrm = torch.exp(0.3 * torch.randn(k, 1, generator=g, device=self.device))
                x = x / x.norm(dim=1, keepdim=True).clamp_min(1e-6) * nrm
            out[s:s + k] = x
        return out


class MnistLike:
    """MNIST8m-shaped (Table I; "less skewness"): 28 x 28 images,
    integer pixels in [0, 255], ~20 % non-zero.  10 classes x 20 prototypes, each
    the sum of 3-5 soft strokes (segments with a Gaussian profile); a sample is
    a prototype under a random shift of up to +-2 px, an intensity jitter and
    pixel noise on the ink, thresholded, scaled to 255 and rounded."""

    SIDE = 28
    PROTOS = 200
    SHIFT = 2

    def __init__(self, dim: int, seed: int, device="cpu"):
        assert dim == self.SIDE * self.SIDE
        g = _gen(seed * 7919 + 17, device)
        self.dim, self.device = dim, device
        S = self.SIDE
        yy, xx = torch.meshgrid(torch.arange(S, device=device, dtype=torch.float32),
                                torch.arange(S, device=device, dtype=torch.float32), indexing="ij")
        protos = torch.zeros(self.PROTOS, S, S, device=device)
        nstroke = torch.randint(3, 6, (self.PROTOS,), generator=g, device=device)
        ends = 5.0 + 18.0 * torch.rand(self.PROTOS, 5, 2, 2, generator=g, device=device)
        for s in range(5):
            a, b = ends[:, s, 0], ends[:, s, 1]                      # [P, 2] (y, x)
            ab = b - a
            t = ((yy[None] - a[:, 0, None, None]) * ab[:, 0, None, None] +
                 (xx[None] - a[:, 1, None, None]) * ab[:, 1, None, None])
            t = (t / (ab * ab).sum(1).clamp_min(1e-6)[:, None, None]).clamp(0, 1)
            py = a[:, 0, None, None] + t * ab[:, 0, None, None]
            px = a[:, 1, None, None] + t * ab[:, 1, None, None]
            d2 = (yy[None] - py) ** 2 + (xx[None] - px) ** 2
            ink = torch.exp(-d2 / (2 * 1.35 ** 2))
            protos += ink * (s < nstroke).float()[:, None, None]
        protos = protos / protos.amax(dim=(1, 2), keepdim=True)
        # every shifted copy of every prototype, flattened: [P * 25, 784]
        pad = torch.nn.functional.pad(protos, (self.SHIFT,) * 4)
        views = []
        for dy in range(2 * self.SHIFT + 1):
            for dx in range(2 * self.SHIFT + 1):
                views.append(pad[:, dy:dy + S, dx:dx + S])
        self.base = torch.stack(views, 1).reshape(-1, dim)

    def sample(self, m: int, seed: int) -> torch.Tensor:
        g = _gen(seed, self.device)
        out = torch.empty(m, self.dim, device=self.device)
        step = 1 << 16
        nb = self.base.shape[0]
        for s in range(0, m, step):
            k = min(step, m - s)
            b = self.base[torch.randint(0, nb, (k,), generator=g, device=self.device)]
            gain = 0.8 + 0.4 * torch.rand(k, 1, generator=g, device=self.device)
            x = b * gain + 0.08 * torch.randn(k, self.dim, generator=g, device=self.device) * (b > 0.1)
            x = torch.where(x > 0.25, x, torch.zeros_like(x))
            out[s:s + k] = torch.clamp(torch.round(x * 255.0), 0, 255)
        return out


def rp_matrix(h: int, dim: int, seed: int, device="cpu") -> torch.Tensor:
    """The random vectors r_1..r_h of §VII's 1-bit random projection (P:467:
    "entries ... iid standard normal"), [h, dim].  Drawn N(0, 1), then rounded
    to multiples of 1/64 and clipped to [-4, 4]: every projection of integer
    pixels is then an exact multiple of 1/64 far below 2^24 / 64, so its sign
    (the code bit) is the same in fp32 in any summation order and in the
    oracle's fp64 (tests check the bound).  Passed to both sides as an input."""
    g = _gen(seed, device)
    r = torch.randn(h, dim, generator=g, device=device, dtype=torch.float32)
    return torch.clamp(torch.round(r * 64.0), -256, 256) / 64.0


def generator_for(cfg: Config, device="cpu"):
    if cfg.kind == "sift":
        return SiftLike(cfg.dim, cfg.seed, device)
    if cfg.kind == "gist":
        return GistLike(cfg.dim, cfg.seed, device)
    if cfg.kind == "glove":
        return ClusteredSkewed(cfg.dim, cfg.seed, 2000, False, device)
    if cfg.kind == "nytimes":
        return ClusteredSkewed(cfg.dim, cfg.seed, 500, True, device)
    if cfg.kind == "mnist":
        return MnistLike(cfg.dim, cfg.seed, device)
    return None


def make_data(cfg: Config, device="cpu", n: Optional[int] = None, nq: Optional[int] = None):
    """(base vectors [n, dim] f32, queries [nq, dim] f32) on `device`."""
    n = cfg.n if n is None else n
    nq = cfg.nq if nq is None else nq
    if cfg.kind == "gauss":
        return gauss(n, cfg.dim, cfg.seed, device), gauss(nq, cfg.dim, cfg.seed + 1, device)
    gen = generator_for(cfg, device)
    return gen.sample(n, cfg.seed), gen.sample(nq, cfg.seed + 1)

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
    # BASELINE.json configs[4] (scale-out): the SIFT1M generator at 100M rows
    # (51.2 GB + a 12.8 GB graph: one B200 holds a replica); s = 500
    "scaleout100m": Config("scaleout100m", 100_000_000, 128, "l2", 32, 10_000, 10, 500, "sift"),
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
    integer pixels in [0, 255], ~20 % non-zero, every sample distinct (MNIST8m
    is MNIST under random deformations).  10 classes x 20 prototypes, each 3-5
    strokes (segments); a sample takes a prototype, jitters every stroke end
    (N(0, 1.2 px)), applies a random similarity transform (rotation +-0.25
    rad, scale 0.85-1.15, shift +-2 px) and a random pen width (1.0-1.6 px),
    renders the strokes with a Gaussian profile, applies an intensity gain,
    thresholds, scales to 255 and rounds."""

    SIDE = 28
    PROTOS = 200
    STROKES = 5

    def __init__(self, dim: int, seed: int, device="cpu"):
        assert dim == self.SIDE * self.SIDE
        g = _gen(seed * 7919 + 17, device)
        self.dim, self.device = dim, device
        self.nstroke = torch.randint(3, self.STROKES + 1, (self.PROTOS,), generator=g, device=device)
        # stroke ends in a centred 18 x 18 box: [P, S, 2 ends, (y, x)]
        self.ends = 5.0 + 18.0 * torch.rand(self.PROTOS, self.STROKES, 2, 2, generator=g,
                                            device=device)
        S = self.SIDE
        yy, xx = torch.meshgrid(torch.arange(S, device=device, dtype=torch.float32),
                                torch.arange(S, device=device, dtype=torch.float32), indexing="ij")
        self.grid = torch.stack([yy.reshape(-1), xx.reshape(-1)], 1)  # [784, 2]

    def _render(self, ends, live, width):
        """ends [k, S, 2, 2] pixel coords, live [k, S] bool, width [k] -> [k, 784] ink."""
        a, b = ends[:, :, 0], ends[:, :, 1]                      # [k, S, 2]
        ab = b - a
        p = self.grid[None, None]                                # [1, 1, 784, 2]
        t = ((p - a[:, :, None]) * ab[:, :, None]).sum(-1)
        t = (t / (ab * ab).sum(-1).clamp_min(1e-6)[:, :, None]).clamp(0, 1)
        near = a[:, :, None] + t[..., None] * ab[:, :, None]     # [k, S, 784, 2]
        d2 = ((p - near) ** 2).sum(-1)                           # [k, S, 784]
        ink = torch.exp(-d2 / (2 * width[:, None, None] ** 2)) * live[:, :, None]
        return ink.amax(1)                                       # [k, 784]

    def sample(self, m: int, seed: int) -> torch.Tensor:
        g = _gen(seed, self.device)
        dev = self.device
        out = torch.empty(m, self.dim, device=dev)
        step = 8192
        c0 = (self.SIDE - 1) / 2.0
        for s in range(0, m, step):
            k = min(step, m - s)
            pid = torch.randint(0, self.PROTOS, (k,), generator=g, device=dev)
            ends = self.ends[pid] + 1.2 * torch.randn(k, self.STROKES, 2, 2, generator=g, device=dev)
            ang = (torch.rand(k, generator=g, device=dev) - 0.5) * 0.5
            scl = 0.85 + 0.3 * torch.rand(k, generator=g, device=dev)
            sh = (torch.rand(k, 2, generator=g, device=dev) - 0.5) * 4.0
            cos, sin = torch.cos(ang) * scl, torch.sin(ang) * scl
            rot = torch.stack([torch.stack([cos, -sin], 1), torch.stack([sin, cos], 1)], 1)
            e = ends - c0
            e = torch.einsum("kij,ksej->ksei", rot, e) + c0 + sh[:, None, None, :]
            live = torch.arange(self.STROKES, device=dev)[None] < self.nstroke[pid][:, None]
            width = 1.0 + 0.6 * torch.rand(k, generator=g, device=dev)
            ink = self._render(e, live, width)
            gain = 0.8 + 0.4 * torch.rand(k, 1, generator=g, device=dev)
            x = ink * gain
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

"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle's tests.

Holds NONE of the method's arithmetic: it only draws 28x28 uint8 images (and seed lists)
with the shape statistics of the paper's workloads (MNIST / Fashion-MNIST, §III-B,
P:93 §IV-B), since the datasets are not available offline.  Recipe: DESIGN.md §6.

  MNIST-shaped   : 3-5 thick Gaussian-blurred strokes in the central 20x20 box, peak 255,
                   target mean intensity ~0.13 (of 255), ~19% nonzero pixels.
  Fashion-shaped : filled union of 2-4 ellipses / rectangles in the central 24x24 box,
                   textured 80..255, target mean ~0.29, ~50% nonzero.
  image k        : class c = k mod 10 prototype, shifted by up to +-2 px, N(0, 25^2) noise on
                   nonzero pixels plus 3% salt pixels, clipped and rounded to uint8.
"""
from __future__ import annotations

import numpy as np

DATA_SEED = 20190325
H = W = 28


def _blur(img: np.ndarray, sigma: float) -> np.ndarray:
    r = max(1, int(np.ceil(2.5 * sigma)))
    x = np.arange(-r, r + 1, dtype=np.float64)
    k = np.exp(-0.5 * (x / sigma) ** 2)
    k /= k.sum()
    pad = np.pad(img, r, mode="constant")
    tmp = np.apply_along_axis(lambda v: np.convolve(v, k, mode="valid"), 1, pad)
    return np.apply_along_axis(lambda v: np.convolve(v, k, mode="valid"), 0, tmp)


def _mnist_prototype(rng: np.random.Generator) -> np.ndarray:
    canvas = np.zeros((H, W), dtype=np.float64)
    yy, xx = np.mgrid[0:H, 0:W]
    n_strokes = int(rng.integers(3, 6))
    pts = rng.uniform(4.5, 23.5, size=(n_strokes + 1, 2))  # central 20x20 box
    for s in range(n_strokes):
        p0, p1 = pts[s], pts[s + 1]
        width = rng.uniform(0.75, 1.1)  # disc radius -> stroke width ~2-3 px after blur
        for u in np.linspace(0.0, 1.0, 40):
            cy, cx = p0 + u * (p1 - p0)
            canvas[(yy - cy) ** 2 + (xx - cx) ** 2 <= width ** 2] = 1.0
    canvas = _blur(canvas, 0.7)
    canvas[canvas < 0.08] = 0.0
    canvas = (canvas / canvas.max()) ** 0.5
    return 255.0 * canvas


def _fashion_prototype(rng: np.random.Generator) -> np.ndarray:
    mask = np.zeros((H, W), dtype=bool)
    yy, xx = np.mgrid[0:H, 0:W]
    for _ in range(int(rng.integers(2, 5))):
        cy, cx = rng.uniform(10.0, 18.0, size=2)
        ry, rx = rng.uniform(4.5, 9.5, size=2)
        if rng.random() < 0.5:
            m = ((yy - cy) / ry) ** 2 + ((xx - cx) / rx) ** 2 <= 1.0
        else:
            m = (np.abs(yy - cy) <= ry) & (np.abs(xx - cx) <= rx)
        mask |= m
    mask[:2, :] = mask[-2:, :] = False
    mask[:, :2] = mask[:, -2:] = False
    texture = 80.0 + 175.0 * _blur(rng.random((H, W)), 1.2)
    texture = 80.0 + (texture - texture.min()) * (175.0 / max(1e-9, texture.max() - texture.min()))
    return np.where(mask, texture, 0.0)


def prototypes(kind: str = "mnist", seed: int = DATA_SEED) -> np.ndarray:
    """10 class prototypes, float64 in [0, 255], shape (10, 28, 28)."""
    rng = np.random.default_rng([seed, 0 if kind == "mnist" else 1])
    make = _mnist_prototype if kind == "mnist" else _fashion_prototype
    return np.stack([make(rng) for _ in range(10)])


def images(n: int, kind: str = "mnist", seed: int = DATA_SEED, start: int = 0) -> np.ndarray:
    """n images (uint8, shape (n, 784)); image k (k = start..start+n-1) has class k mod 10."""
    protos = prototypes(kind, seed)
    out = np.empty((n, H * W), dtype=np.uint8)
    for r in range(n):
        k = start + r
        rng = np.random.default_rng([seed, 2, k])
        img = protos[k % 10]
        dy, dx = rng.integers(-2, 3, size=2)
        img = np.roll(np.roll(img, int(dy), axis=0), int(dx), axis=1)
        nz = img > 0
        img = img + np.where(nz, rng.normal(0.0, 25.0, size=img.shape), 0.0)
        salt = rng.random(img.shape) < 0.03
        img = np.where(salt, rng.uniform(0.0, 255.0, size=img.shape), img)
        out[r] = np.clip(np.rint(img), 0, 255).astype(np.uint8).reshape(-1)
    return out


def labels(n: int, start: int = 0) -> np.ndarray:
    return (np.arange(start, start + n) % 10).astype(np.int32)


def seeds(n: int, base_seed: int = 1, start: int = 0) -> np.ndarray:
    """Per-presentation seeds seed_k = (base_seed << 20) + k."""
    return ((np.uint64(base_seed) << np.uint64(20)) + np.arange(start, start + n, dtype=np.uint64)).astype(np.uint64)


def stats(imgs: np.ndarray) -> dict:
    x = imgs.astype(np.float64) / 255.0
    return dict(mean=float(x.mean()), nonzero=float((imgs > 0).mean()))


def sparse_graph(n_in: int = 784, n_lif: int = 1000, n_syn: int = 10000, bits: int = 8, seed: int = DATA_SEED,
                 recurrent: bool = True):
    """Random synapse list for the Fig. 4 workload (10^3 LIF neurons, 10^4 synapses; R24):
    sources uniform over the n_in input pixels (and, if recurrent, the n_lif neurons), targets uniform over
    the neurons, codes uniform on the 2^bits grid.  CSR by source: (src_off[n_src + 1] int32, tgt u16, q u8).
    Topology only -- none of the method's arithmetic."""
    rng = np.random.default_rng(seed)
    n_src = n_in + (n_lif if recurrent else 0)
    src = rng.integers(0, n_src, size=n_syn)
    tgt = rng.integers(0, n_lif, size=n_syn)
    q = rng.integers(0, 1 << bits, size=n_syn)
    order = np.lexsort((tgt, src))
    src, tgt, q = src[order], tgt[order], q[order]
    off = np.zeros(n_in + n_lif + 1, dtype=np.int32)
    np.add.at(off, src + 1, 1)
    return np.cumsum(off).astype(np.int32), tgt.astype(np.uint16), q.astype(np.uint8)

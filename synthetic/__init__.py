"""Seeded synthetic inputs shared by tests, bench and smoke.

This module holds NO arithmetic of the method (no boundary handling, no
masks, no filtering): it only draws images.  It is the one module both the
oracle side (tests/, bench cpu_baseline) and the CUDA side (via tests/bench)
consume, so both see byte-identical inputs.

Recipe ("angiography-like"; the paper targets
angiography, but ships no data):
  * background 0.55 + a sum of 4 low-frequency cosine plane waves, total
    amplitude <= 0.15;
  * 12 + H/256 vessels: smooth centrelines (sum of 3 random sinusoids around a
    random offset), horizontal or vertical, some spanning only part of the
    image (branches); Gaussian cross-section of radius U(1.5, 8) px darkened
    by U(0.15, 0.4) (contrast agent);
  * additive N(0, 0.02) noise, clipped to [0, 1];
  * u8 variant = round(255 * x).
Frames of a sequence (config C4) reuse the base geometry, scale the vessel
contrast by a bolus curve and shift by up to +-2 px; frame f of a sequence
seeded s uses seed s ^ (f * 0x9E3779B9) for its noise.
Seeds: 2012 * 1000 + config_id (bench/tests use these).
"""
from __future__ import annotations

import math

import torch

SEED_BASE = 2012 * 1000


def config_seed(config_id: int) -> int:
    return SEED_BASE + int(config_id)


def _gen(seed: int, device) -> torch.Generator:
    g = torch.Generator(device=device)
    g.manual_seed(int(seed) & 0x7FFFFFFFFFFFFFFF)
    return g


def _u(g, lo, hi, n=(), device="cpu"):
    return lo + (hi - lo) * torch.rand(n, generator=g, device=device, dtype=torch.float64)


NOISE_BLOCK = 256     # noise is drawn per block of 256 rows, seeded by (seed, frame, block)


def angio(height: int, width: int, seed: int, frame: int = 0, n_frames: int = 1,
          device="cpu", row_range=None) -> torch.Tensor:
    """One float32 angiography-like frame in [0, 1], shape (height, width).

    row_range=(y0, y1) returns only rows [y0, y1) of that same image (used to
    generate row bands in place on each rank); the pixels do not depend on
    the range requested.
    """
    device = torch.device(device)
    H, W = int(height), int(width)
    g = _gen(seed, "cpu")                       # geometry: drawn on CPU (device-independent)
    # background plane waves
    waves = []
    for _ in range(4):
        a = float(_u(g, 0.0, 0.0375))
        fx = float(_u(g, 0.2, 2.5))
        fy = float(_u(g, 0.2, 2.5))
        ph = float(_u(g, 0.0, 2 * math.pi))
        waves.append((a, fx, fy, ph))
    n_vessels = 12 + H // 256
    vessels = []
    for i in range(n_vessels):
        horizontal = bool(torch.rand((), generator=g) < 0.5)
        L, M = (W, H) if horizontal else (H, W)       # along / across extents
        offset = float(_u(g, 0.1, 0.9)) * M
        terms = [(float(_u(g, 0.0, M / 12.0)), float(_u(g, 0.5, 3.0)),
                  float(_u(g, 0.0, 2 * math.pi))) for _ in range(3)]
        radius = float(_u(g, 1.5, 8.0))
        depth = float(_u(g, 0.15, 0.4))
        if i < n_vessels // 2:
            start, stop = 0.0, float(L)
        else:                                          # branch: partial extent
            start = float(_u(g, 0.0, 0.5)) * L
            stop = float(_u(g, 0.5, 1.0)) * L
        vessels.append((horizontal, offset, terms, radius, depth, start, stop))
    # per-frame variation
    if n_frames > 1:
        bolus = 0.35 + 0.65 * math.sin(math.pi * (frame + 0.5) / n_frames)
        sx = round(2.0 * math.sin(2 * math.pi * frame / 17.0))
        sy = round(2.0 * math.cos(2 * math.pi * frame / 23.0))
    else:
        bolus, sx, sy = 1.0, 0, 0
    fseed = seed ^ (int(frame) * 0x9E3779B9)
    y_lo, y_hi = (0, H) if row_range is None else (int(row_range[0]), int(row_range[1]))

    out = torch.empty((y_hi - y_lo, W), dtype=torch.float32, device=device)
    xs = torch.arange(W, device=device, dtype=torch.float32) - sx
    for blk in range(y_lo // NOISE_BLOCK, (y_hi + NOISE_BLOCK - 1) // NOISE_BLOCK):
        r0 = max(y_lo, blk * NOISE_BLOCK)
        r1 = min(y_hi, (blk + 1) * NOISE_BLOCK, H)
        gn = _gen(fseed * 1000003 + blk, device)
        ys = (torch.arange(r0, r1, device=device, dtype=torch.float32) - sy)[:, None]
        img = torch.full((r1 - r0, W), 0.55, device=device, dtype=torch.float32)
        for a, fx, fy, ph in waves:
            img += a * torch.cos(2 * math.pi * (fx * xs[None, :] / W + fy * ys / H) + ph)
        for horizontal, offset, terms, radius, depth, start, stop in vessels:
            along = xs[None, :] if horizontal else ys
            across = ys if horizontal else xs[None, :]
            Lx = W if horizontal else H
            centre = torch.full_like(along, offset)
            for amp, freq, phase in terms:
                centre = centre + amp * torch.sin(2 * math.pi * freq * along / Lx + phase)
            d2 = (across - centre) ** 2
            prof = torch.exp(-d2 / (2.0 * radius * radius))
            inside = ((along >= start) & (along < stop)).to(torch.float32)
            img -= (depth * bolus) * prof * inside
        b0 = blk * NOISE_BLOCK
        noise = torch.randn((min(H, b0 + NOISE_BLOCK) - b0, W), generator=gn, device=device,
                            dtype=torch.float32)[r0 - b0:r1 - b0]
        img += 0.02 * noise
        out[r0 - y_lo:r1 - y_lo] = img.clamp_(0.0, 1.0)
    return out


def angio_frames(n_frames: int, height: int, width: int, seed: int, first: int = 0,
                 count: int | None = None, device="cpu") -> torch.Tensor:
    """Frames [first, first+count) of an n_frames sequence, shape (count, H, W)."""
    count = n_frames - first if count is None else count
    out = torch.empty((count, height, width), dtype=torch.float32, device=device)
    for i in range(count):
        out[i] = angio(height, width, seed, frame=first + i, n_frames=n_frames, device=device)
    return out


def to_u8(img: torch.Tensor) -> torch.Tensor:
    return torch.round(img * 255.0).clamp_(0, 255).to(torch.uint8)


def uniform(height: int, width: int, seed: int, device="cpu") -> torch.Tensor:
    g = _gen(seed, device)
    return torch.rand((height, width), generator=g, device=device, dtype=torch.float32)


def uniform_u8(height: int, width: int, seed: int, device="cpu") -> torch.Tensor:
    g = _gen(seed, device)
    return torch.randint(0, 256, (height, width), generator=g, device=device,
                         dtype=torch.int32).to(torch.uint8)


def levels(height: int, width: int, seed: int, values=(0.0, 0.5, 1.0), block: int = 7,
           device="cpu") -> torch.Tensor:
    """Piecewise-constant image (blocks of random levels) -- step edges."""
    g = _gen(seed, "cpu")
    bh, bw = -(-height // block), -(-width // block)
    idx = torch.randint(0, len(values), (bh, bw), generator=g)
    lv = torch.tensor(values, dtype=torch.float32)[idx]
    img = lv.repeat_interleave(block, 0).repeat_interleave(block, 1)[:height, :width]
    return img.contiguous().to(device)


def checkerboard(height: int, width: int, period: int = 3, lo=0.0, hi=1.0,
                 device="cpu") -> torch.Tensor:
    y = torch.arange(height)[:, None] // period
    x = torch.arange(width)[None, :] // period
    return torch.where((x + y) % 2 == 0, torch.tensor(hi), torch.tensor(lo)).to(
        torch.float32).to(device)


def impulse(height: int, width: int, y: int, x: int, value=1.0, device="cpu") -> torch.Tensor:
    img = torch.zeros((height, width), dtype=torch.float32, device=device)
    img[y, x] = value
    return img


def ramp(height: int, width: int, a=0.01, b=0.02, c=0.1, device="cpu") -> torch.Tensor:
    y = torch.arange(height, dtype=torch.float64)[:, None]
    x = torch.arange(width, dtype=torch.float64)[None, :]
    return (a * x + b * y + c).to(torch.float32).to(device)

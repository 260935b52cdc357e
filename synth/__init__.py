"""Seeded synthetic fields shaped like the paper's datasets (Table 2).

This module holds NO compression arithmetic: it only draws inputs.  Both the
oracle tests and the CUDA parity tests / bench take their inputs from here;
a field is generated once (on any torch device) and the SAME bytes are fed
to both sides.  Recipes follow SURVEY 8(d) and are restated in DESIGN.md
section 6.  Seeds: seed = 1000 + 10 * config + field.
"""
from __future__ import annotations

import math

import torch


def _gen(seed: int, device) -> torch.Generator:
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    return g


def grf(shape, alpha: float, seed: int, device="cpu") -> torch.Tensor:
    """Periodic Gaussian random field with power spectrum P(k) ~ k^-alpha, unit std, float32."""
    g = _gen(seed, device)
    noise = torch.randn(*shape, generator=g, device=device, dtype=torch.float32)
    spec = torch.fft.rfftn(noise)
    del noise
    ks = []
    for d, n in enumerate(shape):
        if d == len(shape) - 1:
            k = torch.fft.rfftfreq(n, device=device) * n
        else:
            k = torch.fft.fftfreq(n, device=device) * n
        view = [1] * len(shape)
        view[d] = k.numel()
        ks.append(k.view(view))
    k2 = ks[0] ** 2
    for k in ks[1:]:
        k2 = k2 + k ** 2
    amp = torch.where(k2 > 0, k2.clamp_min(1e-12) ** (-alpha / 4.0), torch.zeros_like(k2))
    spec = spec * amp
    del amp, k2
    f = torch.fft.irfftn(spec, s=shape)
    del spec
    f = f - f.mean()
    f = f / f.std().clamp_min(1e-30)
    return f.to(torch.float32).contiguous()


# ---- config 1: CESM-ATM 1800x3600 ------------------------------------
def cesm_like(field: int = 0, shape=(1800, 3600), device="cpu") -> torch.Tensor:
    """(0) T-like 250 + 20 g ; (1) cloud-fraction-like clip(0.5 g, 0, 1), ~50% exact zeros."""
    g = grf(shape, 5.0, 1000 + 10 * 1 + field, device)
    if field == 0:
        return (250.0 + 20.0 * g).contiguous()
    return (0.5 * g).clamp(0.0, 1.0).contiguous()


# ---- config 2: Hurricane 100x500x500 ---------------------------------
def hurricane_like(field: int = 0, shape=(100, 500, 500), device="cpu") -> torch.Tensor:
    """(0) U-like vortex wind ~ rho/(0.05+rho^2) * exp(-1.5 z) + 1% noise; (1) QSNOW-like sparse."""
    nz, ny, nx = shape
    z = torch.linspace(0, 1, nz, device=device).view(nz, 1, 1)
    y = torch.linspace(-1, 1, ny, device=device).view(1, ny, 1)
    x = torch.linspace(-1, 1, nx, device=device).view(1, 1, nx)
    cx, cy = 0.1, -0.15
    dy, dx = y - cy, x - cx
    rho = torch.sqrt(dx * dx + dy * dy)
    g = _gen(1000 + 10 * 2 + field, device)
    if field == 0:
        vt = rho / (0.05 + rho * rho)
        u = -vt * (dy / rho.clamp_min(1e-6)) * torch.exp(-1.5 * z) * 30.0
        u = u + 0.01 * u.abs().mean() * torch.randn(nz, ny, nx, generator=g, device=device)
        return u.to(torch.float32).contiguous()
    ring = torch.exp(-((rho - 0.45) ** 2) / 0.01)
    layer = torch.exp(-((z - 0.5) ** 2) / 0.02)
    q = ring * layer * (1.0 + 0.2 * torch.randn(nz, ny, nx, generator=g, device=device))
    return (torch.clamp(q - 0.3, min=0.0) * 1e-3).to(torch.float32).contiguous()


# ---- config 3: NYX 512^3 ----------------------------------------------
def nyx_like(field: int = 0, n: int = 512, device="cpu", seed_offset: int = 0) -> torch.Tensor:
    """(0) baryon-density-like exp(2.5 g); (1) velocity-like g; (2) temperature-like exp(0.7 g).
    seed_offset selects another realisation (one per rank in weak-scaling runs)."""
    g = grf((n, n, n), 4.0, 1000 + 10 * 3 + field + 100000 * seed_offset, device)
    if field == 0:
        return torch.exp(2.5 * g).contiguous()
    if field == 1:
        return (1.0e7 * g).contiguous()
    return (1.0e4 * torch.exp(0.7 * g)).contiguous()


# ---- config 4: HACC 1-D particles ---------------------------------------
HACC_N = 280_953_867


def hacc_like(field: int = 0, n: int = HACC_N, device="cpu") -> torch.Tensor:
    """(0) velocity-like: random walk (step per 4096 particles) x 20 + N(0, 300^2);
    (1) position-like: cell-sorted uniform in [0, 256)."""
    g = _gen(1000 + 10 * 4 + field, device)
    if field == 0:
        nsteps = (n + 4095) // 4096
        walk = torch.cumsum(torch.randn(nsteps, generator=g, device=device) * 20.0, 0)
        bulk = walk.repeat_interleave(4096)[:n]
        return (bulk + 300.0 * torch.randn(n, generator=g, device=device)).to(torch.float32).contiguous()
    ncell = 256 ** 2
    per = (n + ncell - 1) // ncell
    cell = torch.arange(n, device=device, dtype=torch.float64) // per
    cx = (cell % 256)
    frac = torch.rand(n, generator=g, device=device, dtype=torch.float64)
    return (cx + frac).clamp(0, 255.99998).to(torch.float32).contiguous()


# ---- config 5: box-scale and f64 ----------------------------------------
def box_like(shape=(512, 4096, 4096), seed: int = 1050, device="cpu", chunk: int = 16) -> torch.Tensor:
    """Sum of 16 random 3-D plane waves with power-law amplitudes + counter-hash noise, built
    chunk-wise along axis 0 (an FFT at this size is too costly)."""
    g = _gen(seed, torch.device("cpu"))
    kvec = torch.randint(1, 24, (16, 3), generator=g).double()
    phase = torch.rand(16, generator=g).double() * 2 * math.pi
    amp = (kvec.norm(dim=1) ** -1.5)
    nz, ny, nx = shape
    out = torch.empty(shape, dtype=torch.float32, device=device)
    yy = torch.arange(ny, device=device, dtype=torch.float32).view(1, ny, 1) / ny
    xx = torch.arange(nx, device=device, dtype=torch.float32).view(1, 1, nx) / nx
    for z0 in range(0, nz, chunk):
        z1 = min(nz, z0 + chunk)
        zz = torch.arange(z0, z1, device=device, dtype=torch.float32).view(-1, 1, 1) / nz
        acc = torch.zeros((z1 - z0, ny, nx), device=device, dtype=torch.float32)
        for j in range(16):
            kz, ky, kx = (float(v) for v in kvec[j])
            acc += float(amp[j]) * torch.sin(2 * math.pi * (kz * zz + ky * yy + kx * xx) + float(phase[j]))
        idx = (torch.arange(z0 * ny * nx, z1 * ny * nx, device=device, dtype=torch.int64)
               .view(z1 - z0, ny, nx))
        h = (idx * 0x9E3779B1 + seed) & 0xFFFFFFFF
        h = (h ^ (h >> 15)) * 0x2C1B3C6D & 0xFFFFFFFF
        h = h ^ (h >> 12)
        acc += 1e-4 * ((h & 0xFFFF).to(torch.float32) / 65535.0 - 0.5)
        out[z0:z1] = acc
    return out


def miranda_like(shape=(256, 384, 384), device="cpu") -> torch.Tensor:
    """float64 3-D GRF with P(k) ~ k^-11/3 (turbulence-like)."""
    return grf(shape, 11.0 / 3.0, 1051, device).double().contiguous()


def qmcpack_like(shape=(288, 115, 69, 69), device="cpu") -> torch.Tensor:
    """float64 products of sinusoids x Gaussian envelopes (orbital-like)."""
    a, b, c, d = shape
    g = _gen(1052, device)
    i = torch.linspace(0, 1, a, device=device, dtype=torch.float64).view(a, 1, 1, 1)
    x = torch.linspace(-1, 1, b, device=device, dtype=torch.float64).view(1, b, 1, 1)
    y = torch.linspace(-1, 1, c, device=device, dtype=torch.float64).view(1, 1, c, 1)
    z = torch.linspace(-1, 1, d, device=device, dtype=torch.float64).view(1, 1, 1, d)
    f = (torch.sin(3 * math.pi * x + 7 * i) * torch.cos(2 * math.pi * y - 3 * i)
         * torch.sin(math.pi * z + i) * torch.exp(-(x * x + y * y + z * z) / 0.5))
    f = f + 1e-6 * torch.randn(f.shape, generator=g, device=device, dtype=torch.float64)
    return f.contiguous()


# ---- small adversarial / special-value inputs for tests -----------------
def special_values(n: int, seed: int, dtype=torch.float32) -> torch.Tensor:
    """Smooth field salted with +-0, subnormals, +-Inf, NaN, huge values and exact repeats."""
    g = _gen(seed, "cpu")
    t = torch.linspace(0, 20, n, dtype=torch.float64)
    x = torch.sin(t) + 0.01 * torch.randn(n, generator=g, dtype=torch.float64)
    x = x.to(dtype)
    fi = torch.finfo(dtype)
    specials = torch.tensor([0.0, -0.0, fi.tiny / 4, -fi.tiny / 8, float("inf"), float("-inf"),
                             float("nan"), fi.max, -fi.max, 1e30, 1.0], dtype=dtype)
    m = max(1, n // 50)
    pos = torch.randint(0, n, (m,), generator=g)
    which = torch.randint(0, specials.numel(), (m,), generator=g)
    x[pos] = specials[which]
    # a run of exact zeros of both signs and a run of identical values
    if n > 400:
        x[100:200] = 0.0
        x[150:160] = -0.0
        x[300:400] = 3.25
    return x.contiguous()


def offset_field(n: int, seed: int, offset: float, dtype=torch.float32) -> torch.Tensor:
    """Smooth 3-sinusoid mixture + tiny noise + a large constant offset (stresses the R2 guard)."""
    g = _gen(seed, "cpu")
    t = torch.arange(n, dtype=torch.float64)
    x = (torch.sin(t / 97.0) + 0.7 * torch.sin(t / 13.0 + 1.0) + 0.3 * torch.sin(t / 3.1 + 2.0)
         + 1e-4 * torch.randn(n, generator=g, dtype=torch.float64) + offset)
    return x.to(dtype).contiguous()


def random_mix(n: int, seed: int, dtype=torch.float32) -> torch.Tensor:
    """Segments of different character: smooth, noise, constant, steps, sparse spikes."""
    g = _gen(seed, "cpu")
    parts = []
    left = n
    kind = 0
    while left > 0:
        m = min(left, int(torch.randint(1, 700, (1,), generator=g)))
        if kind % 5 == 0:
            p = torch.cumsum(torch.randn(m, generator=g, dtype=torch.float64) * 0.01, 0)
        elif kind % 5 == 1:
            p = torch.randn(m, generator=g, dtype=torch.float64) * 10.0 ** float(torch.randint(-6, 6, (1,), generator=g))
        elif kind % 5 == 2:
            p = torch.full((m,), float(torch.randn(1, generator=g)), dtype=torch.float64)
        elif kind % 5 == 3:
            p = torch.floor(torch.arange(m, dtype=torch.float64) / 37.0) * 0.5
        else:
            p = torch.zeros(m, dtype=torch.float64)
            p[torch.randint(0, m, (max(1, m // 64),), generator=g)] = 1.0
        parts.append(p)
        left -= m
        kind += int(torch.randint(1, 4, (1,), generator=g))
    return torch.cat(parts)[:n].to(dtype).contiguous()

"""Seeded synthetic field generators (harness code; see synth/__init__.py).

All generators return a contiguous float32 torch tensor on ``device``.
Internally they use float32/float64 torch ops; the exact bits differ
between CPU and CUDA builds of torch, so a parity test always generates a
field ONCE and hands the same bytes to both the oracle and the GPU path.
"""
from __future__ import annotations

import math

import torch
import torch.nn.functional as Fnn

# --------------------------------------------------------------------------
# building blocks


def _gen(seed: int, device) -> torch.Generator:
    g = torch.Generator(device=device)
    g.manual_seed(int(seed))
    return g


def _fbm(shape, seed: int, device, base_cells: int = 8, octaves: int = 4,
         gain: float = 0.5) -> torch.Tensor:
    """Smooth Gaussian-like random field: sum of octaves of random lattices,
    each upsampled (multi-)linearly to ``shape``; returns float32 with
    roughly zero mean and unit std."""
    g = _gen(seed, device)
    dims = len(shape)
    mode = {1: "linear", 2: "bilinear", 3: "trilinear"}[dims]
    out = torch.zeros(shape, dtype=torch.float32, device=device)
    amp, total = 1.0, 0.0
    for o in range(octaves):
        cells = base_cells * (2 ** o)
        coarse = [max(2, min(s, math.ceil(s * cells / max(shape)) + 1)) for s in shape]
        lat = torch.randn([1, 1] + coarse, generator=g, device=device, dtype=torch.float32)
        up = Fnn.interpolate(lat, size=list(shape), mode=mode, align_corners=True)[0, 0]
        out.add_(up, alpha=amp)
        total += amp * amp
        amp *= gain
        del up, lat
    out.mul_(1.0 / math.sqrt(total))
    return out


def _uniform(n: int, seed: int, device) -> torch.Tensor:
    return torch.rand(n, generator=_gen(seed, device), device=device, dtype=torch.float32)


# --------------------------------------------------------------------------
# C1: synthetic 1D smooth field (BASELINE.json configs[0])


def smooth1d(n: int = 1 << 20, seed: int = 1, device="cpu") -> torch.Tensor:
    """sum_{m=0..3} 2^-m sin(2 pi f_m i / n + phi_m), f = {3, 11, 37, 101},
    plus uniform noise of 1e-5 x range: smooth, zero-centred."""
    g = _gen(seed, device)
    phases = torch.rand(4, generator=g, device=device, dtype=torch.float64) * (2 * math.pi)
    i = torch.arange(n, device=device, dtype=torch.float64)
    x = torch.zeros(n, device=device, dtype=torch.float64)
    for m, f in enumerate((3, 11, 37, 101)):
        x += (2.0 ** -m) * torch.sin(2 * math.pi * f * i / max(n, 1) + phases[m])
    rng = float(x.max() - x.min()) if n else 0.0
    noise = torch.rand(n, generator=g, device=device, dtype=torch.float64) - 0.5
    x += noise * (1e-5 * rng)
    return x.to(torch.float32).contiguous()


# --------------------------------------------------------------------------
# C2: Hurricane-shaped 100 x 500 x 500 (z, y, x) fields


def hurricane_like(field: str = "U", shape=(100, 500, 500), seed: int = 2,
                   device="cpu") -> torch.Tensor:
    """Isabel-like fields (Table 2: 500x500x100, 13 fields).
    U: Rankine/Holland vortex tangential wind (zero-centred) + 1 % fBm.
    QCLOUD: max(0, fBm - theta) with theta at the 70th percentile -> ~70 %
            exact zeros, contiguous zero regions (zero blocks).
    TC: temperature offset field, ~200..300 K with a lapse rate."""
    Z, Y, X = shape
    if field == "U":
        z = torch.arange(Z, device=device, dtype=torch.float32).view(Z, 1, 1)
        y = torch.arange(Y, device=device, dtype=torch.float32).view(1, Y, 1)
        x = torch.arange(X, device=device, dtype=torch.float32).view(1, 1, X)
        yc, xc = 0.52 * Y, 0.47 * X
        dy, dx = y - yc, x - xc
        r = torch.sqrt(dy * dy + dx * dx) + 1e-3
        rm = 0.05 * max(X, Y)
        vmax = 60.0 * (1.0 - 0.7 * z / max(Z - 1, 1))
        vt = vmax * torch.where(r < rm, r / rm, torch.pow(rm / r, 0.6))
        u = -vt * dy / r + 4.0
        u = u + 1.2 * _fbm(shape, seed, device, base_cells=6)
        return u.contiguous()
    if field == "QCLOUD":
        f = _fbm(shape, seed, device, base_cells=5)
        flat = f.reshape(-1)
        idx = torch.randint(0, flat.numel(), (min(flat.numel(), 1 << 20),),
                            generator=_gen(seed + 101, device), device=device)
        theta = torch.quantile(flat[idx], 0.70)
        return (torch.clamp(f - theta, min=0.0) * 1.5e-3).contiguous()
    if field == "TC":
        z = torch.arange(Z, device=device, dtype=torch.float32).view(Z, 1, 1)
        base = 300.0 - 85.0 * z / max(Z - 1, 1)
        return (base + 3.0 * _fbm(shape, seed, device, base_cells=6)).expand(Z, Y, X).contiguous()
    raise ValueError(field)


# --------------------------------------------------------------------------
# C3: HACC-shaped particle coordinates (1D, n = 280,953,867)


def _morton_decode3(c: torch.Tensor, bits: int):
    x = torch.zeros_like(c)
    y = torch.zeros_like(c)
    z = torch.zeros_like(c)
    for b in range(bits):
        x |= ((c >> (3 * b)) & 1) << b
        y |= ((c >> (3 * b + 1)) & 1) << b
        z |= ((c >> (3 * b + 2)) & 1) << b
    return x, y, z


def hacc_like(n: int = 280_953_867, seed: int = 5, device="cpu", box: float = 256.0,
              grid_bits: int = 6, chunk: int = 1 << 26) -> torch.Tensor:
    """x-coordinates of particles in a [0, box) box, stored in spatially
    coherent (Morton-ordered cell) order with uniform jitter inside each cell:
    locally rough like HACC's coordinate fields (Table 3 CR 3.4-5.2 at 1e-3)."""
    ncell = 1 << (3 * grid_bits)
    cell = box / (1 << grid_bits)
    out = torch.empty(n, dtype=torch.float32, device=device)
    g = _gen(seed, device)
    for s in range(0, n, chunk):
        e = min(n, s + chunk)
        i = torch.arange(s, e, device=device, dtype=torch.int64)
        c = (i * ncell) // max(n, 1)
        cx, _, _ = _morton_decode3(c, grid_bits)
        jitter = torch.rand(e - s, generator=g, device=device, dtype=torch.float32)
        out[s:e] = (cx.to(torch.float32) + jitter) * cell
    return out


# --------------------------------------------------------------------------
# C4: NYX-shaped 512^3 log-normal temperature


def nyx_like(shape=(512, 512, 512), seed: int = 6, device="cpu",
             tmin: float = 2280.975830078125, tmax: float = 4782583.5) -> torch.Tensor:
    """exp(mu + sigma g) with g a smooth Gaussian random field, scaled so the
    field spans the artifact's [min, max]."""
    f = _fbm(shape, seed, device, base_cells=16, octaves=5, gain=0.6)
    lo, hi = f.min(), f.max()
    f.sub_(lo).div_(hi - lo)                       # [0, 1]
    ratio = math.log(tmax / tmin)
    f.mul_(ratio).exp_().mul_(tmin)                # tmin .. tmax, log-normal-like
    return f.contiguous()


# --------------------------------------------------------------------------
# C5: RTM-shaped snapshot set, 36 x 449 x 449 x 235


def _ricker(t: torch.Tensor) -> torch.Tensor:
    a = (math.pi * t) ** 2
    return (1.0 - 2.0 * a) * torch.exp(-a)


def rtm_like(nsnap: int = 36, shape=(449, 449, 235), seed: int = 7, device="cpu",
             out: torch.Tensor | None = None, snaps=None) -> torch.Tensor:
    """Seismic wavefield snapshots (1 per 100 of 3600 steps):
    a Ricker wavefront expanding from a near-surface source with 1/r
    spreading and reflections from 3 layers; EXACTLY 0 ahead of every front
    (and behind it once the pulse has passed: the Ricker tail underflows), so
    the non-zero fraction grows while the front crosses the box (0.3 % at
    t0, 40 % at t14: "sparse early", Fig 22) and falls again
    as it leaves (all zero from ~t25).  Set CR at 1e-3: 44.3 (paper's RTM
    average 42.40, Table 3).
    Shape (nsnap, X, Y, Z) flattened C-order; the set is one 1D array.
    ``snaps``: only these snapshot indices (each identical to its slice of the
    whole set), concatenated in the given order."""
    X, Y, Z = shape
    per = X * Y * Z
    snaps = list(range(nsnap)) if snaps is None else list(snaps)
    if out is None:
        out = torch.empty(len(snaps) * per, dtype=torch.float32, device=device)
    g = _gen(seed, device)
    src = torch.tensor([0.5 * X, 0.5 * Y, 12.0], device=device)
    src = src + torch.rand(3, generator=g, device=device) * 4.0
    layers = [0.35 * Z, 0.6 * Z, 0.85 * Z]
    refl = [0.45, -0.3, 0.25]
    diag = math.sqrt(X * X + Y * Y + Z * Z)
    xs = torch.arange(X, device=device, dtype=torch.float32).view(X, 1, 1)
    ys = torch.arange(Y, device=device, dtype=torch.float32).view(1, Y, 1)
    zs = torch.arange(Z, device=device, dtype=torch.float32).view(1, 1, Z)
    dxy = (xs - src[0]) ** 2 + (ys - src[1]) ** 2
    width = 6.0
    for k, s in enumerate(snaps):
        R = (s + 1) / nsnap * 1.05 * diag
        snap = torch.zeros((X, Y, Z), dtype=torch.float32, device=device)
        r = torch.sqrt(dxy + (zs - src[2]) ** 2) + 1.0
        arg = (r - R) / width
        snap += torch.where(r <= R + 2.5 * width, _ricker(arg) * (200.0 / r), torch.zeros((), device=device))
        for zl, c in zip(layers, refl):
            if R > (zl - float(src[2])):
                zi = 2.0 * zl - src[2]
                ri = torch.sqrt(dxy + (zs - zi) ** 2) + 1.0
                m = (ri <= R + 2.5 * width) & (zs <= zl)
                snap += torch.where(m, c * _ricker((ri - R) / width) * (200.0 / ri), torch.zeros((), device=device))
                del ri, m
        out[k * per:(k + 1) * per] = snap.reshape(-1)
        del snap, r, arg
    return out


# --------------------------------------------------------------------------
# secondary six-dataset shapes


def cesm_like(shape=(1800, 3600), seed: int = 8, device="cpu") -> torch.Tensor:
    lat = torch.linspace(-math.pi / 2, math.pi / 2, shape[0], device=device).view(-1, 1)
    base = 250.0 + 40.0 * torch.cos(lat)
    return (base + 4.0 * _fbm(shape, seed, device, base_cells=12)).expand(*shape).contiguous()


def qmcpack_like(shape=(288, 115, 69, 69), seed: int = 9, device="cpu") -> torch.Tensor:
    O, Z, Y, X = shape
    g = _gen(seed, device)
    out = torch.empty(shape, dtype=torch.float32, device=device)
    z = torch.linspace(-1, 1, Z, device=device).view(Z, 1, 1)
    y = torch.linspace(-1, 1, Y, device=device).view(1, Y, 1)
    x = torch.linspace(-1, 1, X, device=device).view(1, 1, X)
    r2 = x * x + y * y + z * z
    for o in range(O):
        k = torch.rand(3, generator=g, device=device) * 6.0 + 1.0
        out[o] = torch.cos(k[0] * x + k[1] * y + k[2] * z) * torch.exp(-3.0 * r2)
    return out.reshape(-1).contiguous()


# --------------------------------------------------------------------------
# configs (BASELINE.json "configs")

CONFIGS = {
    "c1_smooth1d": dict(n=1 << 20, rel=[1e-4], seed=1),
    "c2_hurricane": dict(shape=(100, 500, 500), fields=["U", "QCLOUD", "TC"], rel=[1e-2, 1e-3, 1e-4], seed=2),
    "c3_hacc": dict(n=280_953_867, rel=[1e-3], seed=5),
    "c4_nyx": dict(shape=(512, 512, 512), rel=[1e-4], seed=6),
    "c5_rtm": dict(nsnap=36, shape=(449, 449, 235), rel=[1e-3], seed=7),
}


# the paper's six datasets (Table 2), one entry per FIELD shape
# (dims per field), REL 1e-2 / 1e-3 / 1e-4 (the paper averages 1e-1 .. 1e-4,
# P:945-948): the bench's six-dataset throughput table
DATASETS = {
    "Hurricane": dict(fields=["U", "QCLOUD", "TC"], dims="100x500x500"),
    "NYX": dict(fields=["temperature"], dims="512x512x512"),
    "QMCPack": dict(fields=["orbitals"], dims="288x115x69x69"),
    "RTM": dict(fields=["t04", "t09", "t14"], dims="449x449x235 (snapshots 4, 9, 14 of 36: the growing front)"),
    "HACC": dict(fields=["x"], dims="280,953,867"),
    "CESM-ATM": dict(fields=["T"], dims="1800x3600"),
}
DATASET_RELS = [1e-2, 1e-3, 1e-4]


def dataset_field(name: str, field: str, device="cpu") -> torch.Tensor:
    """One field of a DATASETS entry as a flat fp32 tensor."""
    if name == "Hurricane":
        return field_for_config("c2_hurricane", device=device, field=field)
    if name == "NYX":
        return field_for_config("c4_nyx", device=device)
    if name == "QMCPack":
        return qmcpack_like(device=device)
    if name == "RTM":
        c = CONFIGS["c5_rtm"]
        return rtm_like(c["nsnap"], c["shape"], c["seed"], device, snaps=[int(field[1:])])
    if name == "HACC":
        return field_for_config("c3_hacc", device=device)
    if name == "CESM-ATM":
        return cesm_like(device=device).reshape(-1)
    raise KeyError(name)


def _scaled(shape, scale: float):
    return tuple(max(2, int(round(s * scale))) for s in shape)


def field_for_config(name: str, device="cpu", scale: float = 1.0, field: str | None = None) -> torch.Tensor:
    """The config's (first, or named) field; ``scale`` < 1 shrinks every
    dimension (tests use small versions of the same recipe)."""
    c = CONFIGS[name]
    if name == "c1_smooth1d":
        return smooth1d(max(1, int(c["n"] * scale)), c["seed"], device)
    if name == "c2_hurricane":
        f = field or "U"
        seed = c["seed"] + c["fields"].index(f)
        return hurricane_like(f, _scaled(c["shape"], scale), seed, device).reshape(-1)
    if name == "c3_hacc":
        return hacc_like(max(1, int(c["n"] * scale)), c["seed"], device)
    if name == "c4_nyx":
        return nyx_like(_scaled(c["shape"], scale), c["seed"], device).reshape(-1)
    if name == "c5_rtm":
        nsnap = c["nsnap"] if scale >= 1.0 else max(2, int(round(c["nsnap"] * scale * 4)))
        return rtm_like(nsnap, _scaled(c["shape"], scale), c["seed"], device)
    raise KeyError(name)

"""Seeded synthetic-input generators shared by the oracle side and the CUDA side.

This module holds NONE of SplitQuant's arithmetic (no quantization, packing,
matmul or normalisation).  It only produces the synthetic weights, activations
and per-layer bit plans that both sides consume, so that an oracle input never
comes from the CUDA path.

Generator (counter based, integer exact, implemented identically in
``synth.cu`` for device-side generation of multi-GB weight sets):

    base   = splitmix64(seed)
    h1     = splitmix64(base + i)            # i = flat element index
    h2     = splitmix64(h1)
    n      = sum of the four 16-bit fields of h1  -  131070   (Irwin-Hall(4),
             mean 0, sd 37837.23, support +-131070: a bounded normal stand-in)
    out    = ((h2 >> 32) % outlier_den) == 0      # ~0.1 % outliers
    value  = fp32(n) * (out ? scale_out : scale)   # ONE IEEE fp32 multiply
    fp16   = round-to-nearest-even(value)

``scale``/``scale_out`` are fp32 constants computed on the host from the
requested standard deviation (sigma / 37837.23, and x10 for outliers), and are
passed unchanged to the device generator, so both sides produce bit-identical
fp16/fp32 values.  The distribution (N(0, 1/K) weights with 0.1 % x10
outliers; N(0, 1) activations) follows SURVEY.md section 8(d) "Synthetic inputs";
the paper uses trained OPT/BLOOM weights, which are out of scope.
"""
from __future__ import annotations

import numpy as np

MASK64 = (1 << 64) - 1
IH4_SD = 37837.2296  # sqrt(4 * (65536**2 - 1) / 12)
OUTLIER_DEN = 1000
OUTLIER_MULT = 10.0

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64_scalar(z: int) -> int:
    z = (z + 0x9E3779B97F4A7C15) & MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def _splitmix64(z: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = z + _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def scales_for(sigma: float, outliers: bool = True) -> tuple[np.float32, np.float32]:
    """fp32 multipliers turning the Irwin-Hall integer into the target sd."""
    s = np.float32(sigma / IH4_SD)
    so = np.float32(sigma * OUTLIER_MULT / IH4_SD) if outliers else s
    return s, so


def _values_f32(seed: int, start: int, count: int, sigma: float, outliers: bool) -> np.ndarray:
    base = np.uint64(splitmix64_scalar(seed & MASK64))
    idx = np.arange(start, start + count, dtype=np.uint64)
    with np.errstate(over="ignore"):
        h1 = _splitmix64(idx + base)
    h2 = _splitmix64(h1)
    m16 = np.uint64(0xFFFF)
    n = ((h1 & m16) + ((h1 >> np.uint64(16)) & m16) + ((h1 >> np.uint64(32)) & m16)
         + (h1 >> np.uint64(48))).astype(np.int64) - 131070
    s, so = scales_for(sigma, outliers)
    mult = np.full(count, s, dtype=np.float32)
    if outliers:
        sel = ((h2 >> np.uint64(32)) % np.uint64(OUTLIER_DEN)) == 0
        mult[sel] = so
    return n.astype(np.float32) * mult  # single IEEE fp32 multiply per element


def fill_f32(seed: int, start: int, count: int, sigma: float = 1.0, outliers: bool = False) -> np.ndarray:
    return _values_f32(seed, start, count, sigma, outliers)


def fill_f16(seed: int, start: int, count: int, sigma: float = 1.0, outliers: bool = False) -> np.ndarray:
    return _values_f32(seed, start, count, sigma, outliers).astype(np.float16)


# ----------------------------------------------------------------------------
# Recipes.  Seeds: weights 1000 + 16*layer + linear,
# activations 1, bit plans 2.
# ----------------------------------------------------------------------------
LINEAR_IDS = {"qkv": 0, "o": 1, "fc1": 2, "fc2": 3}


def weight_seed(layer: int, linear: str | int) -> int:
    lid = LINEAR_IDS[linear] if isinstance(linear, str) else int(linear)
    return 1000 + 16 * layer + lid


def weight_sigma(k: int) -> float:
    return 1.0 / float(np.sqrt(k))


def weight_f16(seed: int, n: int, k: int, rows: np.ndarray | None = None) -> np.ndarray:
    """W [n, k] fp16, element (r, c) = generator index r*k + c.  ``rows`` picks a subset."""
    sig = weight_sigma(k)
    if rows is None:
        return fill_f16(seed, 0, n * k, sig, outliers=True).reshape(n, k)
    out = np.empty((len(rows), k), dtype=np.float16)
    for i, r in enumerate(rows):
        out[i] = fill_f16(seed, int(r) * k, k, sig, outliers=True)
    return out


def bias_f16(seed: int, n: int) -> np.ndarray:
    return fill_f16(seed + 500_000, 0, n, 0.02, outliers=False)


def act_f16(seed: int, m: int, k: int) -> np.ndarray:
    """Activations x [m, k] fp16 ~ N(0, 1)."""
    return fill_f16(seed, 0, m * k, 1.0, outliers=False).reshape(m, k)


def hidden_f32(seed: int, t: int, d: int) -> np.ndarray:
    """Synthetic embeddings x0 [t, d] fp32 ~ N(0, 1) (stand-in for token embeddings)."""
    return fill_f32(seed, 0, t * d, 1.0, outliers=False).reshape(t, d)


def bits_plan(seed: int, n_layers: int, choices=(3, 4, 8, 16), balanced: bool = False) -> np.ndarray:
    """Per-layer bit-widths: the paper's random 'mixed' allocation.

    ``balanced`` = a seeded permutation of equal counts of each choice
    (16 x {3,4,8,16} for 64 layers)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    if balanced:
        reps = -(-n_layers // len(choices))
        arr = np.tile(np.asarray(choices, dtype=np.int32), reps)[:n_layers]
        return rng.permutation(arr).astype(np.int32)
    return rng.choice(np.asarray(choices, dtype=np.int32), size=n_layers).astype(np.int32)


def grid_aligned_weight_f16(seed: int, n: int, k: int, bits: int, group: int = 128) -> tuple[np.ndarray, np.ndarray, np.ndarray, np.ndarray]:
    """Weights that lie exactly on a quantization grid (special case: lossless).

    Returns (W fp16 [n,k], codes u8 [n,k], s fp16 [n,k/g], z fp16 [n,k/g]) with
    W = z + s*c exactly representable in fp16, every group spanning codes 0 and
    2^b - 1 so min/max quantization must reproduce (s, z, c).  Only integer and
    power-of-two arithmetic: s = 2^-e, z = -m * 2^-e chosen so all values are
    exact fp16."""
    rng = np.random.Generator(np.random.PCG64(seed))
    qmax = (1 << bits) - 1
    g = k // group
    e = rng.integers(7, 12, size=(n, g))
    s = np.ldexp(1.0, -e)
    zi = rng.integers(-2 * qmax, qmax, size=(n, g))
    z = zi * s
    c = rng.integers(0, qmax + 1, size=(n, k)).astype(np.int64)
    c[:, ::group] = 0
    c[:, 1::group] = qmax
    w = z.repeat(group, axis=1) + s.repeat(group, axis=1) * c
    w16 = w.astype(np.float16)
    assert np.array_equal(w16.astype(np.float64), w), "grid weights must be fp16-exact"
    return w16, c.astype(np.uint8), s.astype(np.float16), z.astype(np.float16)


def adversarial_weight_f16(seed: int, n: int = 64, k: int = 512) -> np.ndarray:
    """Synthetic weight with the edge cases of the quantizer and the dequantizing kernels (no method
    arithmetic): a constant group, a -0 group, subnormals, +-65504 groups (the dequantized top code
    overflows fp16 unless saturated, R20) in several rows of one 128-row tile, exact
    half-step ties, a linear ramp and a large outlier.  Needs n >= 16, k >= 256."""
    w = weight_f16(seed, n, k).copy()
    w[0, :128] = np.float16(0.5)                                   # constant group
    w[1, 128:256] = np.float16(-0.0)                               # -0 group
    w[1, 130] = np.float16(0.0)
    w[2, :128] = np.float16(6e-8)                                  # subnormal range
    w[2, 5] = np.float16(-6e-8)
    w[3, 0], w[3, 1] = np.float16(65504.0), np.float16(-65504.0)   # extremes (group 0)
    w[4, :128] = (np.arange(128) % 16).astype(np.float16) * np.float16(0.25)  # exact ties for b = 3
    w[5, 128:256] = np.linspace(-1, 1, 128).astype(np.float16)
    w[6, 7] = np.float16(30.0)                                     # outlier
    for r in range(8, min(n, 12)):                                 # extremes in group 1 of more rows
        w[r, 128 + r], w[r, 140 + r] = np.float16(65504.0), np.float16(-65504.0)
    w[12, 200] = np.float16(65504.0)                               # top only: s*qmax + z lands near 65504
    return w

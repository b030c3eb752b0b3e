"""Seeded synthetic inputs shared by the oracle tests, the CUDA parity tests and bench.py.

This module holds NONE of the method's arithmetic: it only draws random numbers with a
counter-free, reproducible recipe (numpy PCG64 streams derived from SeedSequence).  Both
sides of every parity test receive the *same* arrays from here; neither side generates
its own.  The recipe (restated in DESIGN.md "Input recipe"):

* root seed 20190413 (the paper's conference date); per-config seed = root + 1000*cfg#;
* each tensor gets its own stream keyed by (seed, name) so adding a tensor never perturbs
  another one;
* weights ~ U(-1/sqrt(H), 1/sqrt(H)) (contractive dynamics);
* MI-LSTM alpha/beta ~ U(0.5, 1.5) for tests;
* states ~ U(-0.5, 0.5); inputs ~ U(-1, 1); upstream gradients ~ N(0, 1);
* tokens ~ Zipf(s=1) over a symbol set, i.i.d. (PTB / enwik8-like frequency skew);
* sentence lengths (bucketed workloads) ~ round(LogNormal(ln 20, 0.5)) clipped to [2, 83]:
  its quintiles (13, 18, 23, 30) sit near the paper's PTB bucket edges 13/18/24/30 with a tail
  to the 83 maximum.
"""
from __future__ import annotations

import zlib

import numpy as np

ROOT_SEED = 20190413


def config_seed(cfg_index: int) -> int:
    """Per-config seed: root + 1000*cfg# (cfg# is 1-based as in SURVEY §8 'cfg1..cfg5')."""
    return ROOT_SEED + 1000 * int(cfg_index)


def rng(seed: int, key: str) -> np.random.Generator:
    """An independent PCG64 stream for tensor `key` under `seed`."""
    ss = np.random.SeedSequence([int(seed) & 0xFFFFFFFF, zlib.crc32(key.encode())])
    return np.random.Generator(np.random.PCG64(ss))


def uniform(seed: int, key: str, shape, lo: float, hi: float) -> np.ndarray:
    return rng(seed, key).uniform(lo, hi, size=shape).astype(np.float64)


def normal(seed: int, key: str, shape, scale: float = 1.0) -> np.ndarray:
    return (rng(seed, key).standard_normal(size=shape) * scale).astype(np.float64)


def zipf_tokens(seed: int, key: str, shape, vocab: int, n_symbols: int | None = None) -> np.ndarray:
    """i.i.d. tokens with p(rank r) ∝ 1/r over `n_symbols` ranks, mapped into [0, vocab).

    With n_symbols < vocab (char LM: 205 distinct bytes of 256), ranks are scattered over
    the vocabulary by a fixed seeded permutation so unused ids exist, as in real byte data.
    """
    n = vocab if n_symbols is None else int(n_symbols)
    g = rng(seed, key)
    p = 1.0 / np.arange(1, n + 1, dtype=np.float64)
    p /= p.sum()
    ranks = g.choice(n, size=shape, p=p)
    perm = rng(seed, key + "/perm").permutation(vocab)[:n]
    return perm[ranks].astype(np.int32)


def weights(seed: int, shapes: dict, hidden: int, overrides: dict | None = None) -> dict:
    """Draw every parameter in `shapes` (name -> shape) from U(±1/sqrt(hidden)).

    `overrides` maps name -> (lo, hi) for parameters with another recipe (e.g. MI-LSTM
    alpha/beta ~ U(0.5, 1.5)).
    """
    bound = 1.0 / np.sqrt(hidden)
    out = {}
    for name, shp in shapes.items():
        lo, hi = (overrides or {}).get(name, (-bound, bound))
        out[name] = uniform(seed, "param/" + name, shp, lo, hi)
    return out


def ptb_like_lengths(seed: int, key: str, n: int, lo: int = 2, hi: int = 83) -> np.ndarray:
    """n mini-batch lengths ~ round(LogNormal(mu = ln 20, sigma = 0.5)), clipped to [lo, hi]."""
    x = rng(seed, key).lognormal(np.log(20.0), 0.5, size=n)
    return np.clip(np.rint(x), lo, hi).astype(np.int64)

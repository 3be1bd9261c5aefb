"""Philox4x32-10 (Salmon et al., SC'11) and the dropout keep-mask recipe.

The paper does not discuss the RNG of dropout; it relies on
``torch.utils.checkpoint`` restoring the RNG state for recompute (P:217,
§V).  Reading R-B: a counter-based generator whose counter is a
pure function of (element, site, step) makes replay exact by construction.

Pinned by: Random123 known-answer vectors (tests/golden/philox_kat.txt),
keep-rate statistics.
"""
from __future__ import annotations

import numpy as np

M0 = np.uint64(0xD2511F53)
M1 = np.uint64(0xCD9E8D57)
W0 = 0x9E3779B9
W1 = 0xBB67AE85
MASK32 = np.uint64(0xFFFFFFFF)

KIND_ATTN_PROBS = 0
KIND_ATTN_OUT = 1
KIND_FFN_OUT = 2
KIND_EMB = 3
KIND_HEAD = 4
LAYER_NONE = 0xFFF


def philox4x32_10(c0, c1, c2, c3, k0: int, k1: int):
    """Vectorised Philox4x32 with 10 rounds; all words are uint32 held in uint64."""
    c0 = np.asarray(c0, np.uint64) & MASK32
    c1 = np.asarray(c1, np.uint64) & MASK32
    c2 = np.asarray(c2, np.uint64) & MASK32
    c3 = np.asarray(c3, np.uint64) & MASK32
    c0, c1, c2, c3 = np.broadcast_arrays(c0, c1, c2, c3)
    key0, key1 = k0 & 0xFFFFFFFF, k1 & 0xFFFFFFFF
    for r in range(10):
        if r:
            key0 = (key0 + W0) & 0xFFFFFFFF
            key1 = (key1 + W1) & 0xFFFFFFFF
        p0 = M0 * c0                      # < 2^64, exact in uint64
        p1 = M1 * c2
        hi0, lo0 = p0 >> np.uint64(32), p0 & MASK32
        hi1, lo1 = p1 >> np.uint64(32), p1 & MASK32
        c0, c1, c2, c3 = (hi1 ^ c1 ^ np.uint64(key0), lo1,
                          hi0 ^ c3 ^ np.uint64(key1), lo0)
    return c0, c1, c2, c3


def site_word(kind: int, layer: int = LAYER_NONE, rank: int = 0) -> int:
    """site = (rank << 16) | (layer_field << 4) | kind  (DESIGN R-B)."""
    return ((rank & 0xFFFF) << 16) | ((layer & 0xFFF) << 4) | (kind & 0xF)


def keep_threshold(p: float) -> int:
    """keep iff r < floor((1-p) * 2^32), computed once in fp64."""
    return int(np.floor((1.0 - p) * 4294967296.0))


def uniform_words(n_elems: int, seed: int, site: int, step: int) -> np.ndarray:
    """The 32-bit random word of element e, e = 0..n_elems-1:
    counter = (e>>2 lo, e>>2 hi, site, step), key = (seed lo, seed hi), lane e&3."""
    e = np.arange(n_elems, dtype=np.uint64)
    n = e >> np.uint64(2)
    lane = (e & np.uint64(3)).astype(np.int64)
    r = philox4x32_10(n & MASK32, n >> np.uint64(32), site, step,
                      seed & 0xFFFFFFFF, (seed >> 32) & 0xFFFFFFFF)
    words = np.stack(r, axis=0)           # [4, n]
    return words[lane, np.arange(n_elems)]


def keep_mask(n_elems: int, p: float, seed: int, site: int, step: int) -> np.ndarray:
    """Boolean keep mask (True = kept) for a tensor flattened in the documented
    element order of its site."""
    if p <= 0.0:
        return np.ones(n_elems, bool)
    return uniform_words(n_elems, seed, site, step) < np.uint64(keep_threshold(p))

"""Two-pattern stimuli (p1 -> p2) packed as uint32 words.

Layout (the C-ABI's): p1, p2 are uint32 [n_pairs][ceil(n_pi/32)],
bit (i % 32) of word (i // 32) is primary input i.  Pair j launches every PI
whose bit differs at t = 0 (reading C2).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass
class Stimuli:
    n_pi: int
    p1: np.ndarray     # uint32 [n_pairs][words]
    p2: np.ndarray     # uint32 [n_pairs][words]

    @property
    def n_pairs(self) -> int:
        return int(self.p1.shape[0])

    @property
    def words(self) -> int:
        return int(self.p1.shape[1])

    def bits(self, which: int) -> np.ndarray:
        """Unpacked uint8 [n_pairs][n_pi] of p1 (which=1) or p2 (which=2)."""
        w = self.p1 if which == 1 else self.p2
        b = np.unpackbits(w.view(np.uint8).reshape(w.shape[0], -1), axis=1, bitorder="little")
        return b[:, :self.n_pi]

    def subset(self, pairs) -> "Stimuli":
        pairs = np.asarray(pairs)
        return Stimuli(self.n_pi, self.p1[pairs].copy(), self.p2[pairs].copy())


def pack_bits(bits: np.ndarray) -> np.ndarray:
    """uint8 [n][n_pi] -> uint32 [n][ceil(n_pi/32)]."""
    n, n_pi = bits.shape
    words = (n_pi + 31) // 32
    pad = np.zeros((n, words * 32), dtype=np.uint8)
    pad[:, :n_pi] = bits
    packed = np.packbits(pad, axis=1, bitorder="little")
    return packed.view(np.uint32).reshape(n, words).copy()


def make_stimuli(seed: int, n_pi: int, n_pairs: int, toggle: float = 0.5) -> Stimuli:
    """p1 uniform over {0,1}^n_pi; p2 = p1 xor Bernoulli(toggle) mask."""
    rng = np.random.default_rng(seed)
    b1 = (rng.random((n_pairs, n_pi)) < 0.5).astype(np.uint8)
    flip = (rng.random((n_pairs, n_pi)) < toggle).astype(np.uint8)
    return Stimuli(n_pi, pack_bits(b1), pack_bits(b1 ^ flip))


def exhaustive_pairs(n_pi: int) -> Stimuli:
    """All 2^n_pi x 2^n_pi ordered pairs (c17: 1024 pairs), p1-major."""
    v = np.arange(1 << n_pi)
    bits = ((v[:, None] >> np.arange(n_pi)[None, :]) & 1).astype(np.uint8)
    i1, i2 = np.meshgrid(v, v, indexing="ij")
    return Stimuli(n_pi, pack_bits(bits[i1.ravel()]), pack_bits(bits[i2.ravel()]))

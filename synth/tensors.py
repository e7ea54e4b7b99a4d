"""Seeded synthetic tensors for the tenants' layers.

* weights ~ N(0, 1/fan_in) (float32 here; the product side rounds to bf16 when
  the layer is bf16, and the oracle then reads the GPU's own rounded values);
* folded-BN per-channel scale ~ U(0.5, 1.5), shift ~ N(0, 0.1);
* activations / inputs ~ N(0, 1);
* token ids ~ U[0, 30522).

Seeds: weights 1000 + tenant index, traces {1, 2, 3}.  Values never affect
timing; they only have to be the same on both sides of a parity check.
"""
from __future__ import annotations

import numpy as np


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def weight(g: np.random.Generator, shape, fan_in: int) -> np.ndarray:
    return (g.standard_normal(size=shape) / np.sqrt(float(fan_in))).astype(np.float32)


def bn_scale(g: np.random.Generator, c: int) -> np.ndarray:
    return g.uniform(0.5, 1.5, size=c).astype(np.float32)


def bn_shift(g: np.random.Generator, c: int) -> np.ndarray:
    return (0.1 * g.standard_normal(size=c)).astype(np.float32)


def bias(g: np.random.Generator, c: int) -> np.ndarray:
    return (0.1 * g.standard_normal(size=c)).astype(np.float32)


def activation(g: np.random.Generator, shape) -> np.ndarray:
    return g.standard_normal(size=shape).astype(np.float32)


def token_ids(g: np.random.Generator, n: int, vocab: int = 30522) -> np.ndarray:
    return g.integers(0, vocab, size=n).astype(np.int32)

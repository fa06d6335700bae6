"""Pins for the oracle's hash / priority / label contract (DESIGN.md §3 H).

The paper never states its RNG, so the contract is ours; it is
pinned here against published test vectors (tests/golden/hash_vectors.txt) and
mathematical facts (bijectivity via an independently derived inverse, uniformity of
the RAND label "chosen uniformly at random", Alg 2 l.3).
"""
import os

import numpy as np
import pytest

import oracle as O

GOLD = os.path.join(os.path.dirname(__file__), "golden", "hash_vectors.txt")


def _vectors():
    for line in open(GOLD):
        if line.strip() and not line.startswith("#"):
            name, x, y = line.split()[:3]
            yield name, int(x, 16), int(y, 16)


@pytest.mark.parametrize("name,x,y", list(_vectors()))
def test_published_vectors(name, x, y):
    f = {"mix64": O.mix64, "fmix32": O.fmix32}[name]
    assert f(x) == y


def _inv_xorshift(h, s, bits):
    # inverse of h ^= h >> s on `bits`-bit words: iterate the fixed point
    x = h
    for _ in range(bits // s + 1):
        x = h ^ (x >> s)
    return x


def _fmix32_inverse(h):
    """Inverse of MurmurHash3 fmix32 derived from its published constants only."""
    M = 2**32
    h = _inv_xorshift(h, 16, 32)
    h = (h * pow(0xC2B2AE35, -1, M)) % M
    h = _inv_xorshift(h, 13, 32)
    h = (h * pow(0x85EBCA6B, -1, M)) % M
    h = _inv_xorshift(h, 16, 32)
    return h


def test_fmix32_is_a_bijection():
    rng = np.random.default_rng(0)
    for x in list(rng.integers(0, 2**32, 2000)) + [0, 1, 2**32 - 1, 0x80000000]:
        x = int(x)
        assert _fmix32_inverse(O.fmix32(x)) == x


def test_pv_has_no_ties_on_a_block():
    # pv is fmix32(v ^ Klo) ^ Khi: injective; check a 2^16 block for every seed class
    for seed in (1, 42, 2**64 - 1):
        vals = {O.pv(seed, v) for v in range(1 << 12)}
        assert len(vals) == 1 << 12


def test_stream_keys_differ_by_tag_and_seed():
    keys = {O.stream_key(s, t) for s in (0, 1, 42, 2**64 - 1) for t in (1, 2, 3)}
    assert len(keys) == 12


def test_pe_is_symmetric_in_wrapper_and_depends_on_both_ends():
    s = 42
    assert O.pe(s, 3, 9) == O.pe(s, 9, 3)
    assert len({O.pe(s, 0, w) for w in range(1, 200)}) == 199


@pytest.mark.parametrize("p", [1, 2, 4, 10, 64, 65535])
def test_rand_label_uniform(p):
    """Alg 2 l.3: each vertex picks one of p parts uniformly at random.
    Chi-square on 200k vertices (p <= 64); range check always."""
    n = 200_000 if p <= 64 else 20_000
    labels = O.classes(np.zeros(n + 1, np.int64), np.zeros(0, np.int32), "rand", p, 42)
    assert labels.max() < p
    if p == 1:
        assert (labels == 0).all()
        return
    if p > 64:
        return
    cnt = np.bincount(labels, minlength=p)
    exp = n / p
    chi2 = ((cnt - exp) ** 2 / exp).sum()
    # dof = p-1; mean p-1, sd sqrt(2(p-1)); 6 sd bound
    assert chi2 < (p - 1) + 6 * np.sqrt(2 * (p - 1))

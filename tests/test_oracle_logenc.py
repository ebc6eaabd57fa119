"""Pins for the oracle's log encoding (Fig. 1; NEXT-2, R19, R24)."""
import numpy as np
import pytest

import oracle


def test_figure1_example():
    # Fig. 1: five integers, x_max = 123 -> 7 bits, two 32-bit containers, 160 -> 64 bits
    x = [123, 5, 64, 99, 17]
    w, b = oracle.log_encode(x)
    assert b == 7 and w.size == 2 and 32 * w.size == 64 and 32 * len(x) == 160
    assert oracle.log_decode(w, 5, b).tolist() == x


def test_bits_is_bit_width():
    # R19: ceil(log2 x_max) is one short at powers of two; bit_width is the count of bits
    assert [oracle.log_bits(v) for v in (0, 1, 2, 3, 4, 123, 127, 128, 2**32 - 1, 2**32, 2**64 - 1)] == \
        [0, 1, 2, 2, 3, 7, 7, 8, 32, 33, 64]
    for v in range(1, 5000):
        b = oracle.log_bits(v)
        assert 2 ** (b - 1) <= v < 2 ** b


def test_hand_built_containers():
    w, b = oracle.log_encode([1, 2, 3], 2)
    assert b == 2 and w.tolist() == [0b111001]
    # value 4 (bits 28..34) spans two containers
    w, b = oracle.log_encode([123, 0, 0, 0, 127], 7)
    assert w.tolist() == [(123 | (127 << 28)) & 0xFFFFFFFF, 127 >> 4]
    w, b = oracle.log_encode([2**40 + 3], 41)
    assert w.tolist() == [3, 2**8]
    w, b = oracle.log_encode([0, 0, 0])
    assert b == 0 and w.size == 0 and oracle.log_decode(w, 3, 0).tolist() == [0, 0, 0]


@pytest.mark.parametrize("b", [1, 5, 7, 13, 23, 26, 31, 32, 33, 47, 64])
def test_layout_matches_numpy_unpackbits_and_round_trips(b):
    rng = np.random.default_rng(b)
    n = 257
    hi = 2**b if b < 64 else 2**64
    x = rng.integers(0, hi, size=n, dtype=np.uint64) if b < 64 else \
        rng.integers(0, 2**63, size=n, dtype=np.uint64) * 2 + 1
    x[0] = (hi - 1) if b < 64 else np.uint64(2**64 - 1)
    w, bb = oracle.log_encode(x)
    assert bb == b and w.size == (n * b + 31) // 32
    # independent statement of the layout: little-endian bit stream of the values
    bits = np.unpackbits(x.astype("<u8").view(np.uint8).reshape(n, 8), axis=1, bitorder="little")[:, :b].reshape(-1)
    bits = np.concatenate([bits, np.zeros(32 * w.size - bits.size, dtype=np.uint8)])
    want = np.packbits(bits, bitorder="little").view("<u4")
    assert np.array_equal(w, want)
    assert np.array_equal(oracle.log_decode(w, n, b), x)

"""Pins for the input generator."""
import numpy as np

from synth.payload import op_seed, payload, splitmix_word


def test_splitmix64_reference_vector():
    # Published SplitMix64 test vector (Vigna's splitmix64.c, seed 1234567):
    # the counter form z = s + (i+1)*golden equals the sequential state update.
    expect = [6457827717110365317, 3203168211198807973, 9817491932198370423,
              4593380528125082431, 16408922859458223821]
    assert [splitmix_word(1234567, i) for i in range(5)] == expect
    w = payload(1234567, 40).view("<u8")
    assert [int(x) for x in w] == expect


def test_payload_offsets_and_tail():
    full = payload(99, 1000)
    for off in [0, 1, 7, 8, 9, 500]:
        for n in [0, 1, 3, 8, 13, 200]:
            assert np.array_equal(payload(99, n, off), full[off:off + n])
    # truncation: first 5 bytes are the low bytes of word 0 (little endian)
    w0 = splitmix_word(99, 0)
    assert list(payload(99, 5)) == [(w0 >> (8 * i)) & 0xFF for i in range(5)]


def test_op_seed():
    assert op_seed(1000, 3) == 1000 * 1_000_003 + 3
    assert op_seed(2**63, 1) == (2**63 * 1_000_003 + 1) % 2**64

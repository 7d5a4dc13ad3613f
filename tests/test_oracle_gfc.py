"""Pins of the GFC compression oracle (oracle/gfc.py).

* the hand-derived byte streams of tests/golden/gfc_examples.json (a worked example of the
  paper's residual/prefix rules, with a negative residual, a capped zero-residual count and
  a ragged last micro-chunk);
* closed forms of the compressed size: all-zero data, constant data (the uniform
  superposition), which the encoding rules fix without running the encoder;
* losslessness: decompress(compress(x)) reproduces every bit pattern (NaN payloads, -0.0,
  infinities, denormals, random patterns, simulated states), at ragged sizes;
* the size bound max_bytes.
"""
import json
import os

import numpy as np
import pytest

from oracle import gfc

GOLD = os.path.join(os.path.dirname(__file__), "golden", "gfc_examples.json")


def _golden():
    return json.load(open(GOLD))["cases"]


@pytest.mark.parametrize("case", _golden(), ids=lambda c: c["name"])
def test_golden_streams(case):
    words = np.array([int(h, 16) for h in case["words_hex"]], dtype=np.uint64)
    want = b"".join(bytes.fromhex(h) * r for h, r in case["stream_parts"])
    stream, off = gfc.compress(words.view(np.float64), case["seg_len"])
    assert stream == want
    assert off.tolist() == case["offsets"]
    back = gfc.decompress(stream, off, len(words), case["seg_len"])
    assert np.array_equal(back.view(np.uint64), words)


@pytest.mark.parametrize("n,seg", [(32, 32), (1000, 64), (4096, 1024), (4097, 1024), (7, 32)])
def test_zero_data_size_closed_form(n, seg):
    # every residual is 0 -> nibble 7 + one zero byte per value; per segment of c values:
    # ceil-per-micro-chunk nibble bytes + c payload bytes, padded to 16
    stream, off = gfc.compress(np.zeros(n), seg)
    want = 0
    for s in range(0, n, seg):
        c = min(seg, n - s)
        full, rest = divmod(c, 32)
        b = full * (16 + 32) + ((rest + 1) // 2 + rest if rest else 0)
        want += b + (-b) % 16
    assert len(stream) == want
    assert set(stream) == {0x00, 0x77} | ({0x07} if n % 2 else set())


def test_constant_data_size_closed_form():
    # uniform superposition of 10 qubits: every double is 2^-5 = 0x3FA0000000000000 (re) or 0
    # (im). First micro-chunk per segment: 16 values of 8 bytes (re), 16 of 1 byte (im);
    # later micro-chunks: all residuals 0 -> 48 bytes.
    n_amp = 1 << 10
    psi = np.full(n_amp, 2.0 ** -5, dtype=np.complex128)
    seg = 256
    stream, off = gfc.compress(psi, seg)
    per_seg = (16 + 16 * 8 + 16 * 1) + (seg // 32 - 1) * 48
    per_seg += (-per_seg) % 16
    assert len(stream) == (2 * n_amp // seg) * per_seg
    assert np.array_equal(gfc.decompress(stream, off, 2 * n_amp, seg), psi.view(np.float64))


def test_roundtrip_special_patterns():
    special = np.array([0x0, 0x8000000000000000, 0x7FF0000000000000, 0xFFF0000000000000,
                        0x7FF8000000000001, 0xFFFFFFFFFFFFFFFF, 0x1, 0x000FFFFFFFFFFFFF,
                        0x7FEFFFFFFFFFFFFF, 0x3FF0000000000000], dtype=np.uint64)
    rng = np.random.default_rng(7)
    words = rng.choice(special, size=777).astype(np.uint64)
    stream, off = gfc.compress(words.view(np.float64), 96)
    back = gfc.decompress(stream, off, len(words), 96)
    assert np.array_equal(back.view(np.uint64), words)
    assert len(stream) <= gfc.max_bytes(len(words), 96)


@pytest.mark.parametrize("n,seg", [(1, 32), (33, 32), (2049, 256), (5000, 4096)])
def test_roundtrip_random_bits(n, seg):
    rng = np.random.default_rng(n)
    words = rng.integers(0, 2 ** 63, size=n, dtype=np.uint64) * np.uint64(2) + rng.integers(0, 2, size=n, dtype=np.uint64)
    stream, off = gfc.compress(words.view(np.float64), seg)
    assert len(stream) <= gfc.max_bytes(n, seg)
    assert int(off[-1]) == len(stream) and all(int(o) % 16 == 0 for o in off)
    assert np.array_equal(gfc.decompress(stream, off, n, seg).view(np.uint64), words)


def test_roundtrip_simulated_states():
    from oracle import statevector as sv
    from workloads import circuits as wc
    for c in (wc.qaoa(10, 2, seed=1), wc.iqp(10), wc.qft(10, x=37), wc.gs(2, 5)):
        psi = sv.simulate(c.qasm())
        stream, off = gfc.compress(psi, 512)
        assert np.array_equal(gfc.decompress(stream, off, 2 * psi.size, 512), psi.view(np.float64))


def test_max_bytes_is_reached_by_incompressible_data():
    # residuals with a set top byte in every value (alternating sign) use all 8 payload bytes
    n, seg = 256, 128
    words = np.where(np.arange(n) % 64 < 32, 0x7F00000000000000, 0x0100000000000000).astype(np.uint64)
    stream, _ = gfc.compress(words.view(np.float64), seg)
    assert len(stream) == gfc.max_bytes(n, seg)

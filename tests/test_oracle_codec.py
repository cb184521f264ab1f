"""Pins for oracle/codec.py (PAPER §IV-B/C, Eq. 6–9, Eq. 11–12)."""

import json
import math
import os

import numpy as np
import pytest

from oracle import codec

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _n(k):
    with open(os.path.join(GOLDEN, "keys.json")) as f:
        d = json.load(f)[k]
    return int(d["p"], 16) * int(d["q"], 16)


def test_eq7_literal_at_alpha_half():
    """At alpha = 1/2 the normalised reading c11 IS literal Eq. 7: q = (m + 1/2)(2^r - 1)."""
    rng = np.random.default_rng(0)
    for rho in (8, 16, 30):
        for m in rng.uniform(-0.5, 0.5, 2000).astype(np.float32):
            e = float(m) + 0.5                                   # Eq. 6
            assert codec.quantize(float(m), 0.5, rho) == round(e * ((1 << rho) - 1))  # Eq. 7


def test_hand_worked_pack_example():
    """alpha = 1/2, r = 30, b = 2 (w = 32, the L432 setting), S = 3 values [-0.5, 0, 0.5]:
    q = [0, round(0.5 * (2^30 - 1)) = 2^29 (half-to-even), 2^30 - 1];  Eq. 9 puts q0 in the top
    slot: Z = 0 * 2^64 + 2^29 * 2^32 + (2^30 - 1) = 2^61 + 2^30 - 1."""
    z = codec.pack([-0.5, 0.0, 0.5], 0.5, 30, 2, 3)
    assert z == [(1 << 61) + (1 << 30) - 1]
    assert codec.unpack_sums(z, 3, 30, 2, 3) == [0, 1 << 29, (1 << 30) - 1]
    x = codec.unpack(z, 3, 0.5, 30, 2, 3, 1)
    assert x[0] == -0.5 and x[2] == 0.5 and 0 < x[1] < 1e-9


def test_eq8_padding_bits_are_zero():
    """Eq. 8: each w-bit slot is [b zero bits][q]: the top b bits of every slot are zero."""
    vals = list(np.random.default_rng(1).uniform(-1, 1, 63 * 3).astype(np.float32))
    for z in codec.pack(vals, 1.0, 29, 3, 63):
        for i in range(63):
            assert (z >> (i * 32 + 29)) & 0b111 == 0


def test_clamp_and_nan():
    assert codec.quantize(float("nan"), 1.0, 29) == codec.quantize(0.0, 1.0, 29)
    assert codec.quantize(5.0, 1.0, 29) == (1 << 29) - 1
    assert codec.quantize(-7.0, 1.0, 29) == 0
    assert codec.quantize(float("inf"), 0.5, 30) == (1 << 30) - 1


def test_tail_slots_zero():
    z = codec.pack([0.5] * 5, 0.5, 30, 2, 3)
    assert len(z) == 2
    assert z[1] & ((1 << 32) - 1) == 0  # third slot of the last plaintext is empty


@pytest.mark.parametrize("k,lit,corr", [(1024, 32, 31), (2048, 64, 63), (4096, 128, 127)])
def test_compression_ratio_l263(k, lit, corr):
    """L263: r + b = 32 gives 32x / 64x / 128x at k = 1024 / 2048 / 4096 (paper-literal
    capacity floor(k/w)); the no-wrap capacity floor((k-1)/w) gives 31 / 63 / 127 (reading c16)."""
    assert codec.slot_capacity_literal(k, 32) == lit
    assert codec.slot_capacity(k, 32) == corr
    n_values = lit * corr * 10
    assert codec.compression_ratio(n_values, lit) == lit
    assert codec.compression_ratio(n_values, corr) == corr
    assert codec.compression_ratio(n_values + 1, corr) < corr  # Eq. 11 "<= k/w" with a tail
    assert codec.psu(n_values, 32, k, lit) == 1.0                # Eq. 12 equality case
    assert codec.psu(n_values, 32, k, corr) == pytest.approx(corr * 32 / k)
    assert codec.num_plaintexts(1 << 20, 63) == 16645            # C2's M


def test_no_wrap_capacity_and_literal_wraps():
    """Reading c16: with S = floor((bits(n)-1)/w) slots and P <= 2^b summands the aggregate of
    P maximal plaintexts stays below n; the literal S = k/w can exceed n."""
    n = _n("2048")
    rho, b, w = 29, 3, 32
    qmax = (1 << rho) - 1
    for slots in (codec.slot_capacity(n.bit_length(), w), codec.slot_capacity_literal(2048, w)):
        agg = sum((1 << b) * qmax << ((slots - 1 - i) * w) for i in range(slots))
        if slots == 63:
            assert agg < n
        else:
            assert agg >= n


def test_roundtrip_error_bound_single():
    """|dequant(quant(x)) - x| <= alpha/(2^r - 1) (half a quantum) + one binary32 rounding."""
    rng = np.random.default_rng(2)
    for alpha, rho in ((1.0, 29), (0.5, 30), (1.0, 44)):
        vals = rng.uniform(-alpha, alpha, 3000).astype(np.float32)
        z = codec.pack(list(vals), alpha, rho, 32 - rho if rho < 32 else 64 - rho, 1)
        back = codec.unpack(z, len(vals), alpha, rho, 32 - rho if rho < 32 else 64 - rho, 1, 1)
        for x, y in zip(vals, back):
            bound = alpha / ((1 << rho) - 1) + abs(float(x)) * 2.0 ** -24 + 2.0 ** -149
            assert abs(float(x) - y) <= bound


def test_aggregate_error_bound():
    """Sum of cnt quantised values dequantised with cnt: |x - sum| <= cnt*alpha/(2^r-1) + rounding."""
    rng = np.random.default_rng(3)
    cnt, alpha, rho, b, S = 8, 1.0, 29, 3, 63
    clients = [rng.normal(0, 0.05, 500).clip(-1, 1).astype(np.float32) for _ in range(cnt)]
    packed = [codec.pack(list(c), alpha, rho, b, S) for c in clients]
    agg = [sum(col) for col in zip(*packed)]  # plaintext sums (what Dec(prod Enc) returns)
    back = codec.unpack(agg, 500, alpha, rho, b, S, cnt)
    exact = np.sum(np.array(clients, dtype=np.float64), axis=0)
    for x, y in zip(exact, back):
        assert abs(x - y) <= cnt * alpha / ((1 << rho) - 1) + abs(x) * 2.0 ** -24 + 1e-12


def test_per_plaintext_counts():
    z = codec.pack([0.25, -0.25, 0.5, 0.0], 1.0, 44, 20, 2)
    s = [z[0] * 3, z[1] * 5]  # plaintext 0 summed 3 times, plaintext 1 five times
    x = codec.unpack(s, 4, 1.0, 44, 20, 2, [3, 5])
    assert x == pytest.approx([0.75, -0.75, 2.5, 0.0], abs=1e-9)


def test_overflow_bits():
    assert [codec.overflow_bits(p) for p in (1, 2, 3, 4, 8, 9, 1 << 20)] == [0, 1, 2, 2, 3, 4, 20]

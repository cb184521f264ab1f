"""Encoding-quantisation and batch compression, §IV-B/§IV-C (ORACLE — test infrastructure).

Paper passages:

* L215 (Eq. 6): e = m + alpha, for a real gradient m in [-alpha, alpha].
* L219–L221 (Eq. 7): q = e * (2^r - 1), "r bits to amplify" (this build writes rho for r).
* L223–L226 (Eq. 8): z = [b zero bits][q], b = ceil(log2 p) overflow bits for p participants.
* L258–L260 (Eq. 9): floor(k / (r + ceil(log2 p))) values packed into one plaintext,
  Z = [00..][q0][00..][q1]...[00..][q_{n-1}].
* L263: with r + b = 32, 32x / 64x / 128x compression at k = 1024 / 2048 / 4096.
* L297 (§V-A): after decryption the plaintext is "unpacked, unquantified and decoded".
* L321–L323 (Eq. 11, 12): compression ratio and plaintext-space utilisation (PSU).

Readings: Eq. 7 is normalised to q = round_half_even((clamp(m)+alpha) * sigma)
with sigma = (2^rho - 1)/(2 alpha) in binary64, identical to literal Eq. 7 at alpha = 1/2 (c11);
NaN -> 0.0, out-of-range values clamp (c13); dequantisation x = S/sigma - cnt*alpha in binary64
then rounded to binary32 (c14); slot capacity floor((bits(n)-1)/w) so a packed sum stays below
n (c16); q0 is the most significant slot, Z = sum_i q_i 2^((S-1-i) w), tail slots zero (c17).
"""

from __future__ import annotations

import math
from typing import List, Optional, Sequence, Union

import numpy as np


def sigma(alpha: float, qbits: int) -> float:
    """Quantisation scale (2^rho - 1) / (2 alpha), one binary64 division (reading c11)."""
    return float((1 << qbits) - 1) / (2.0 * alpha)


def quantize(x: float, alpha: float, qbits: int) -> int:
    """One value through Eq. 6 and Eq. 7 in binary64, step by step."""
    if x != x:  # NaN -> 0.0 (reading c13)
        x = 0.0
    xc = min(max(float(x), -alpha), alpha)  # clamp to [-alpha, alpha] (L215 domain)
    e = xc + alpha                           # Eq. 6
    q = round(e * sigma(alpha, qbits))       # Eq. 7, round half to even (reading c11)
    return min(max(q, 0), (1 << qbits) - 1)


def slot_capacity(n_bits: int, slot_bits: int) -> int:
    """Slots per plaintext: floor((bits(n) - 1) / w) (reading c16 of PAPER L258)."""
    return (n_bits - 1) // slot_bits


def slot_capacity_literal(key_bits: int, slot_bits: int) -> int:
    """The paper-literal count floor(k / w) of PAPER L258 (may wrap mod n; comparison only)."""
    return key_bits // slot_bits


def num_plaintexts(n_values: int, slots: int) -> int:
    """ceil(N / S): plaintexts (= ciphertexts) after batch compression (Eq. 11 denominator)."""
    return -(-n_values // slots)


def compression_ratio(n_values: int, slots: int) -> float:
    """Eq. 11 (garbled fraction restored per reading c20): N / ceil(N / S)."""
    return n_values / num_plaintexts(n_values, slots)


def psu(n_values: int, slot_bits: int, key_bits: int, slots: int) -> float:
    """Eq. 12: N * w / (k * ceil(N / S))."""
    return n_values * slot_bits / (key_bits * num_plaintexts(n_values, slots))


def pack(values: Sequence[float], alpha: float, qbits: int, pad_bits: int, slots: int) -> List[int]:
    """Quantise and pack (Eq. 6–9): plaintext j = sum_{i<S} q_{jS+i} * 2^((S-1-i) w).

    ``values`` are binary32 numbers (Python floats holding binary32 values).  Slot i of
    plaintext j holds value jS+i; slots past the end are zero (reading c17).
    """
    w = qbits + pad_bits
    out = []
    for j in range(num_plaintexts(len(values), slots)):
        z = 0
        for i in range(slots):
            t = j * slots + i
            if t < len(values):
                z += quantize(values[t], alpha, qbits) << ((slots - 1 - i) * w)
        out.append(z)
    return out


def unpack_sums(plaintexts: Sequence[int], n_values: int, qbits: int, pad_bits: int,
                slots: int) -> List[int]:
    """The exact w-bit slot integers Sum_i, in value order (inverse of Eq. 9's layout)."""
    w = qbits + pad_bits
    mask = (1 << w) - 1
    out = []
    for t in range(n_values):
        j, i = divmod(t, slots)
        out.append((plaintexts[j] >> ((slots - 1 - i) * w)) & mask)
    return out


def dequantize(s: int, cnt: int, alpha: float, qbits: int) -> float:
    """x = Sum / sigma - cnt * alpha in binary64, rounded once to binary32 (reading c14).

    cnt is the number of quantised values summed into the slot (each carried +alpha, Eq. 6).
    """
    v = float(s) / sigma(alpha, qbits) - float(cnt) * alpha
    return float(np.float32(v))


def unpack(plaintexts: Sequence[int], n_values: int, alpha: float, qbits: int, pad_bits: int,
           slots: int, summands: Union[int, Sequence[int]] = 1) -> List[float]:
    """Unpack, unquantise and decode.  ``summands`` is a scalar count, or one
    count per plaintext (e.g. the population of a histogram bin)."""
    sums = unpack_sums(plaintexts, n_values, qbits, pad_bits, slots)
    out = []
    for t, s in enumerate(sums):
        cnt = summands if isinstance(summands, int) else int(summands[t // slots])
        out.append(dequantize(s, cnt, alpha, qbits))
    return out


def overflow_bits(participants: int) -> int:
    """b = ceil(log2 p) (Eq. 8 context)."""
    return max(0, math.ceil(math.log2(participants))) if participants > 1 else 0

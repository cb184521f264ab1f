"""Philox4x32-10 counter-based generator and the Paillier r drawn from it (ORACLE).

PAPER L209 (§IV-A3): "we develop a random number generator for large integers ...,
assigning a random number generator for each thread".  The paper names no generator; this
build fixes Philox4x32-10 (Salmon et al., SC'11, the Random123 library) so that r is a pure
function of (seed, element index) — reading c4 in DESIGN.md §3.  The generator itself is
pinned by the Random123 known-answer vectors (tests/golden/philox_kat.txt).
"""

from __future__ import annotations

from typing import List, Tuple

_M0 = 0xD2511F53
_M1 = 0xCD9E8D57
_W0 = 0x9E3779B9
_W1 = 0xBB67AE85
_MASK = 0xFFFFFFFF


def philox4x32_10(ctr: Tuple[int, int, int, int], key: Tuple[int, int]) -> Tuple[int, int, int, int]:
    """Ten Philox-4x32 rounds (Random123 ``philox4x32_R(10, ...)``)."""
    c0, c1, c2, c3 = (v & _MASK for v in ctr)
    k0, k1 = (v & _MASK for v in key)
    for rnd in range(10):
        if rnd:
            k0 = (k0 + _W0) & _MASK
            k1 = (k1 + _W1) & _MASK
        p0 = _M0 * c0
        p1 = _M1 * c2
        hi0, lo0 = p0 >> 32, p0 & _MASK
        hi1, lo1 = p1 >> 32, p1 & _MASK
        c0, c1, c2, c3 = (hi1 ^ c1 ^ k0, lo1, hi0 ^ c3 ^ k1, lo0)
    return (c0, c1, c2, c3)


def philox_words(seed: int, index: int, nwords: int) -> List[int]:
    """``nwords`` 32-bit words for element ``index``: key = (seed lo, seed hi),
    counter = (index lo, index hi, block j, 0), word 4j+t = output t of block j (reading c4)."""
    key = (seed & _MASK, (seed >> 32) & _MASK)
    words: List[int] = []
    j = 0
    while len(words) < nwords:
        words.extend(philox4x32_10((index & _MASK, (index >> 32) & _MASK, j, 0), key))
        j += 1
    return words[:nwords]


def draw_r(n: int, seed: int, index: int, pt_words: int) -> int:
    """Encryption randomness r for element ``index`` (r in Z*_{n^2}; reading c3/c4).

    r = (little-endian value of ``pt_words`` Philox words) with every bit >= bits(n)-1 cleared,
    so 0 <= r < 2^(bits(n)-1) <= n; r = 0 is replaced by 1.  gcd(r, n) != 1 is not rejected
    (probability ~2^(1-k/2) for real keys); r^n mod n^2 depends only on r mod n (reading c3).
    """
    words = philox_words(seed, index, pt_words)
    r = 0
    for i, w in enumerate(words):
        r |= w << (32 * i)
    r &= (1 << (n.bit_length() - 1)) - 1
    return r if r else 1

"""Generic modular arithmetic and textbook RSA (ORACLE — test infrastructure).

PAPER Table I (L236–L256) and §IV-D (L269–L284): `mod_mul(values1, values2, n)` = values1 *
values2 % n (L245, L279), `mod_pow(x, p, n)` = x^p % n (L246, L280), and RSA::key_gen / encrypt /
decrypt / mul (L247–L251, L281–L284) with "multiplicative homomorphism" (L209).  Written as the
plain definitions (Python ints; `pow` is the library primitive).  RSA follows the textbook scheme
(Rivest–Shamir–Adleman): n = p q, e = 65537, d = e^-1 mod lcm(p-1, q-1), Enc(m) = m^e mod n,
Dec(c) = c^d mod n, Mul(c1, c2) = c1 c2 mod n.  Pinned in tests/test_oracle_modarith.py.

Table I's fundamentals over unsigned `words`-limb integers: add/sub
modulo 2^(32 words) with the carry/borrow out, the full product, division with remainder
(b = 0: quotient 2^(32 words) - 1 and remainder a, the convention of the binary division), mod,
and the modular inverse by the extended Euclidean algorithm written out (0 when none exists).
"""

from __future__ import annotations

import math
import random
from typing import Tuple

from . import paillier


def mod_mul(a: int, b: int, n: int) -> int:
    """Table I mod_mul."""
    return a * b % n


def mod_pow(x: int, e: int, n: int) -> int:
    """Table I mod_pow."""
    return pow(x, e, n)


def rsa_keygen(key_bits: int, seed: int, e: int = 65537) -> Tuple[int, int, int, int]:
    """RSA::key_gen: returns (n, e, d, p) with p the larger prime."""
    rng = random.Random(seed)
    half = key_bits // 2
    while True:
        p = paillier.random_prime(half, rng)
        q = paillier.random_prime(half, rng)
        if p == q:
            continue
        lam = math.lcm(p - 1, q - 1)
        if math.gcd(e, lam) != 1 or (p * q).bit_length() != key_bits:
            continue
        return p * q, e, pow(e, -1, lam), max(p, q)


def rsa_encrypt(n: int, e: int, m: int) -> int:
    """RSA::encrypt: m^e mod n."""
    return pow(m, e, n)


def rsa_decrypt(n: int, d: int, c: int) -> int:
    """RSA::decrypt: c^d mod n."""
    return pow(c, d, n)


def rsa_mul(n: int, c1: int, c2: int) -> int:
    """RSA::mul: the multiplicative homomorphism c1 c2 mod n."""
    return c1 * c2 % n


# ----------------------------------------------------------------------------- Table I fundamentals
def mp_add(a: int, b: int, words: int) -> Tuple[int, int]:
    """Table I add: ((a + b) mod 2^(32 words), carry out)."""
    s = a + b
    return s % (1 << (32 * words)), s >> (32 * words)


def mp_sub(a: int, b: int, words: int) -> Tuple[int, int]:
    """Table I sub: ((a - b) mod 2^(32 words), borrow = [a < b])."""
    return (a - b) % (1 << (32 * words)), 1 if a < b else 0


def mp_mul(a: int, b: int) -> int:
    """Table I mul: the full product."""
    return a * b


def mp_divmod(a: int, b: int, words: int) -> Tuple[int, int]:
    """Table I div / mod: (floor(a / b), a mod b); b = 0 -> (2^(32 words) - 1, a)."""
    if b == 0:
        return (1 << (32 * words)) - 1, a
    return a // b, a % b


def mod_inv(x: int, n: int) -> int:
    """Table I mod_inv: x^-1 mod n by the extended Euclidean algorithm; 0 if n < 2 or
    gcd(x, n) != 1."""
    if n < 2:
        return 0
    r0, r1 = n, x % n
    s0, s1 = 0, 1          # invariant: s_i x = r_i (mod n)
    while r1 != 0:
        q = r0 // r1
        r0, r1 = r1, r0 - q * r1
        s0, s1 = s1, s0 - q * s1
    if r0 != 1:
        return 0
    return s0 % n

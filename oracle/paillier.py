"""Paillier cryptosystem, written out as PAPER.md §III-B defines it (ORACLE — test infrastructure).

Every big integer is a Python ``int``.  Nothing here is fast; everything here is checkable
against the paper by eye.

Paper passages (``/root/reference/PAPER.md``):

* L89  (§III-B, key generation): primes p, q; n = p*q; lambda = lcm(p-1, q-1); g in Z*_{n^2}
  with gcd(n, L(g^lambda mod n^2)) = 1; L(x) = (x-1)/n; public key (g, n), private (p, q).
* L90–L92 (§III-B, Eq. 3): E(m) = g^m * r^n mod n^2 (the text's "q^m" is a garble of g^m).
* L94–L96 (§III-B, Eq. 4): D(c) = L(c^lambda mod n^2) / L(g^lambda mod n^2) mod n.
* L116–L119 (§III-B, Eq. 5): E(m1) * E(m2) = E(m1 + m2)  -> homomorphic add is c1*c2 mod n^2.
* L246/L280 (Table I mod_pow) and L209 ("multiplicative homomorphism"): scalar multiply is
  c^e mod n^2 (reading c19).
* L71 (§III-A, Fig. 2 aggregation) generalised: a segmented product of ciphertexts mod n^2.

Readings: g = n + 1 (c1), r in [1, 2^(bits(n)-1)) drawn by philox.draw_r (c3/c4),
p and q of key_bits/2 bits each with the top two bits set so bits(n) = key_bits (c5).
"""

from __future__ import annotations

import math
import random
from typing import Iterable, List, Optional, Sequence, Tuple

# ----------------------------------------------------------------------------- key generation

_SMALL_PRIMES = [x for x in range(3, 2000) if all(x % d for d in range(2, int(x ** 0.5) + 1))]


def is_probable_prime(x: int, rng: random.Random, rounds: int = 40) -> bool:
    """Miller–Rabin (PAPER L209 names Miller–Rabin [46] for the primes of key generation)."""
    if x < 2:
        return False
    for sp in [2] + _SMALL_PRIMES:
        if x == sp:
            return True
        if x % sp == 0:
            return False
    d, s = x - 1, 0
    while d % 2 == 0:
        d //= 2
        s += 1
    for _ in range(rounds):
        a = rng.randrange(2, x - 1)
        y = pow(a, d, x)
        if y in (1, x - 1):
            continue
        for _ in range(s - 1):
            y = y * y % x
            if y == x - 1:
                break
        else:
            return False
    return True


def miller_rabin_bases(x: int, bases: Iterable[int]) -> bool:
    """Miller–Rabin with the given bases: True iff x passes every round.
    Write x - 1 = d 2^s with d odd; x passes base a iff a^d = 1 or a^(d 2^r) = x - 1 for some
    r < s (mod x).  A base with a mod x in {0} is treated as the round a^d mod x computes."""
    if x < 3 or x % 2 == 0:
        return x == 2
    d, s = x - 1, 0
    while d % 2 == 0:
        d //= 2
        s += 1
    for a in bases:
        y = pow(a, d, x)
        if y == 1 or y == x - 1:
            continue
        for _ in range(s - 1):
            y = y * y % x
            if y == x - 1:
                break
        else:
            return False
    return True


def random_prime(bits: int, rng: random.Random) -> int:
    """A random ``bits``-bit prime with its top two bits and its low bit set (reading c5)."""
    while True:
        cand = rng.getrandbits(bits) | (3 << (bits - 2)) | 1
        if is_probable_prime(cand, rng):
            return cand


def keygen(key_bits: int, seed: int) -> Tuple[int, int]:
    """Paillier key generation, deterministic in ``seed``.

    Returns the private key (p, q) with p > q; the public key is n = p*q and g = n + 1
    (reading c1).  bits(p) = bits(q) = key_bits/2 and bits(n) = key_bits (reading c5).
    """
    if key_bits % 2 or key_bits < 16:
        raise ValueError("key_bits must be even and >= 16")
    rng = random.Random(seed)
    half = key_bits // 2
    while True:
        p = random_prime(half, rng)
        q = random_prime(half, rng)
        if p == q:
            continue
        n = p * q
        if n.bit_length() != key_bits:
            continue
        if math.gcd(n, (p - 1) * (q - 1)) != 1:
            continue
        return (max(p, q), min(p, q))


# ----------------------------------------------------------------------------- the scheme


def L(x: int, n: int) -> int:
    """L(x) = (x - 1) / n."""
    return (x - 1) // n


def public_g(n: int) -> int:
    """g = n + 1 (reading c1 of PAPER L89; the north star fixes g)."""
    return n + 1


def encrypt(n: int, m: int, r: int) -> int:
    """E(m) = g^m * r^n mod n^2 (Eq. 3), g = n + 1."""
    n2 = n * n
    return pow(public_g(n), m, n2) * pow(r, n, n2) % n2


def decrypt(p: int, q: int, c: int) -> int:
    """D(c) = L(c^lambda mod n^2) / L(g^lambda mod n^2) mod n (Eq. 4).

    "Division" by L(g^lambda mod n^2) is multiplication by its inverse mod n (it is invertible
    by the gcd condition of L89), i.e. mu = L(g^lambda mod n^2)^-1 mod n.
    """
    n = p * q
    n2 = n * n
    lam = math.lcm(p - 1, q - 1)
    mu = pow(L(pow(public_g(n), lam, n2), n), -1, n)
    return L(pow(c, lam, n2), n) * mu % n


def add(n: int, c1: int, c2: int) -> int:
    """Homomorphic addition: E(m1) * E(m2) mod n^2 = E(m1 + m2) (Eq. 5)."""
    return c1 * c2 % (n * n)


def scalar_mul(n: int, c: int, e: int) -> int:
    """Homomorphic scalar multiply: E(m)^e mod n^2 = E(e*m) (mod_pow; reading c19)."""
    return pow(c, e, n * n)


def reduce_segments(n: int, cs: Sequence[int], offsets: Sequence[int],
                    idx: Optional[Sequence[int]] = None) -> List[int]:
    """out[j] = prod_{t in [offsets[j], offsets[j+1])} cs[idx[t]] mod n^2; empty product = 1.

    The server-side aggregation of Fig. 2 as repeated Eq. 5 (L118).
    """
    n2 = n * n
    out = []
    for j in range(len(offsets) - 1):
        acc = 1
        for t in range(offsets[j], offsets[j + 1]):
            acc = acc * cs[idx[t] if idx is not None else t] % n2
        out.append(acc)
    return out


# ----------------------------------------------------------------------------- limb helpers


def to_limbs(x: int, words: int) -> List[int]:
    """Little-endian 32-bit limbs (base 2^w, w = 32), exactly ``words`` of them."""
    if x < 0 or x >> (32 * words):
        raise ValueError("value does not fit in %d limbs" % words)
    return [(x >> (32 * i)) & 0xFFFFFFFF for i in range(words)]


def from_limbs(limbs: Iterable[int]) -> int:
    v = 0
    for i, w in enumerate(limbs):
        v |= (int(w) & 0xFFFFFFFF) << (32 * i)
    return v

"""Pins for oracle/modarith.py (Table I mod_mul / mod_pow, RSA)."""

import math
import random

import pytest

from oracle import modarith


def test_mod_pow_against_repeated_multiplication():
    rng = random.Random(1)
    for _ in range(200):
        n = rng.randrange(3, 1 << 40) | 1
        x, e = rng.randrange(n), rng.randrange(0, 60)
        acc = 1 % n
        for _ in range(e):
            acc = acc * x % n
        assert modarith.mod_pow(x, e, n) == acc


def test_fermat_and_euler():
    p = (1 << 127) - 1  # Mersenne prime
    rng = random.Random(2)
    for _ in range(10):
        a = rng.randrange(2, p)
        assert modarith.mod_pow(a, p - 1, p) == 1
    n = 1009 * 2003
    phi = 1008 * 2002
    for a in range(2, 200):
        if math.gcd(a, n) == 1:
            assert modarith.mod_pow(a, phi, n) == 1


def test_mod_mul_small_exhaustive():
    for n in (7, 15, 16, 31):
        for a in range(n):
            for b in range(n):
                assert modarith.mod_mul(a, b, n) == (a * b) % n


@pytest.mark.parametrize("bits", [64, 512])
def test_rsa_roundtrip_and_homomorphism(bits):
    n, e, d, p = modarith.rsa_keygen(bits, 3)
    q = n // p
    assert p * q == n and n.bit_length() == bits and (e * d) % math.lcm(p - 1, q - 1) == 1
    rng = random.Random(4)
    for _ in range(20):
        m1, m2 = rng.randrange(n), rng.randrange(n)
        c1, c2 = modarith.rsa_encrypt(n, e, m1), modarith.rsa_encrypt(n, e, m2)
        assert modarith.rsa_decrypt(n, d, c1) == m1
        assert modarith.rsa_decrypt(n, d, modarith.rsa_mul(n, c1, c2)) == m1 * m2 % n


def test_rsa_tiny_exhaustive():
    # textbook example p = 61, q = 53, e = 17, d = 413 (lambda = 780): all m round-trip
    n, e, d = 61 * 53, 17, pow(17, -1, math.lcm(60, 52))
    assert d == 413
    for m in range(n):
        assert modarith.rsa_decrypt(n, d, modarith.rsa_encrypt(n, e, m)) == m


# ----------------------------------------------------------------------------- Table I fundamentals
def test_mp_add_sub_identities():
    rng = random.Random(7)
    for words in (1, 3, 64):
        R = 1 << (32 * words)
        for a, b in [(0, 0), (R - 1, 1), (R - 1, R - 1), (1, R - 1)] + [(rng.randrange(R), rng.randrange(R))
                                                                         for _ in range(50)]:
            s, c = modarith.mp_add(a, b, words)
            assert s + c * R == a + b and 0 <= s < R and c in (0, 1)
            d, br = modarith.mp_sub(a, b, words)
            assert d - br * R == a - b and 0 <= d < R and br in (0, 1)
            # sub undoes add modulo R
            assert modarith.mp_sub(s, b, words)[0] == a


def test_mp_divmod_euclid_property():
    rng = random.Random(8)
    for words in (1, 2, 33):
        R = 1 << (32 * words)
        for _ in range(100):
            a, b = rng.randrange(R), rng.randrange(1, R) >> rng.randrange(0, 32 * words)
            b = max(b, 1)
            q, r = modarith.mp_divmod(a, b, words)
            assert a == q * b + r and 0 <= r < b
        assert modarith.mp_divmod(12345, 0, words) == (R - 1, 12345)
    # exhaustive tiny: repeated subtraction
    for a in range(60):
        for b in range(1, 13):
            q, r = 0, a
            while r >= b:
                r -= b
                q += 1
            assert modarith.mp_divmod(a, b, 1) == (q, r)


def test_mod_inv_brute_force_small_moduli():
    for n in range(1, 70):
        for x in range(0, 3 * n):
            inv = [y for y in range(1, n) if (x * y) % n == 1 % n] if n >= 2 else []
            want = inv[0] if inv else 0
            assert modarith.mod_inv(x, n) == want, (x, n)


def test_mod_inv_large_and_key_use():
    rng = random.Random(9)
    for _ in range(50):
        n = rng.randrange(2, 1 << 512)
        x = rng.randrange(0, 1 << 520)
        y = modarith.mod_inv(x, n)
        if math.gcd(x, n) == 1:
            assert 1 <= y < n and (x * y) % n == 1 % n
        else:
            assert y == 0
    # RSA private exponent d = e^-1 mod lambda (an even modulus), the textbook example
    assert modarith.mod_inv(17, math.lcm(60, 52)) == 413

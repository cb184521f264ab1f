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

"""Pins for oracle/paillier.py — checks against what the paper and the mathematics fix,
never against a retyped copy of the oracle's own formula ("pins")."""

import json
import math
import os
import random

import pytest

from oracle import paillier, philox, montgomery

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _keys():
    with open(os.path.join(GOLDEN, "keys.json")) as f:
        d = json.load(f)
    return {k: (int(v["p"], 16), int(v["q"], 16)) for k, v in d.items()}


KEYS = _keys()


def _fermat_prime(x, bases=(2, 3, 5, 7, 11, 13)):
    return all(pow(b, x - 1, x) == 1 for b in bases)


# ----------------------------------------------------------------------------- key generation

def test_keygen_toy_primes_trial_division():
    # brute-force primality of small generated primes (independent of Miller-Rabin)
    for seed in range(20):
        p, q = paillier.keygen(24, seed)
        for x in (p, q):
            assert all(x % d for d in range(2, int(math.isqrt(x)) + 1))
            assert x.bit_length() == 12 and (x >> 10) == 3 and x & 1
        assert (p * q).bit_length() == 24 and p > q


@pytest.mark.parametrize("k", ["1024", "2048", "3072", "4096"])
def test_golden_keys_are_valid(k):
    p, q = KEYS[k]
    bits = int(k)
    assert p != q and p > q
    assert p.bit_length() == q.bit_length() == bits // 2
    assert (p * q).bit_length() == bits
    assert _fermat_prime(p) and _fermat_prime(q)
    assert math.gcd(p * q, (p - 1) * (q - 1)) == 1


def test_golden_keys_reproducible():
    p, q = paillier.keygen(1024, 0xF1B0 + 1024)
    assert (p, q) == KEYS["1024"]


def test_miller_rabin_rejects_carmichael_and_composites():
    rng = random.Random(1)
    for c in (561, 1105, 1729, 2465, 2821, 6601, 8911, 41041, 62745, 3215031751):
        assert not paillier.is_probable_prime(c, rng)
    assert paillier.is_probable_prime((1 << 127) - 1, rng)  # Mersenne prime M127
    assert not paillier.is_probable_prime((1 << 127) + 1, rng)


# ----------------------------------------------------------------------------- toy-key brute force

def test_toy16_all_messages_roundtrip():
    """Every m < n for n = 251*241 = 60,491: Dec(Enc(m)) = m (Eq. 3, Eq. 4)."""
    p, q = KEYS["toy16"]
    n = p * q
    rng = random.Random(7)
    for m in range(n):
        r = rng.randrange(1, n)
        while math.gcd(r, n) != 1:
            r = rng.randrange(1, n)
        assert paillier.decrypt(p, q, paillier.encrypt(n, m, r)) == m


def test_toy9_exhaustive_add_and_scalar():
    """All (a, b) for n = 17*19 = 323: Dec(E(a)E(b)) = a+b, Dec(E(a)^b) = a*b mod n (Eq. 5)."""
    p, q = KEYS["toy9"]
    n = p * q
    n2 = n * n
    rng = random.Random(9)
    units = [r for r in range(1, n) if math.gcd(r, n) == 1]
    enc = [paillier.encrypt(n, a, rng.choice(units)) for a in range(n)]
    # decryption table: brute force inverse of the encryption map restricted to our ciphertexts
    lam = math.lcm(p - 1, q - 1)
    for a in range(n):
        ca = enc[a]
        for b in range(n):
            s = paillier.add(n, ca, enc[b])
            assert paillier.decrypt(p, q, s) == (a + b) % n
            e = paillier.scalar_mul(n, ca, b)
            assert paillier.decrypt(p, q, e) == (a * b) % n
    assert lam == 144


def test_toy_encryption_is_injective_in_m():
    """For fixed r, Enc(., r) is a bijection Z_n -> residues (Paillier's permutation property)."""
    p, q = KEYS["toy9"]
    n = p * q
    seen = {paillier.encrypt(n, m, 5) for m in range(n)}
    assert len(seen) == n


# ----------------------------------------------------------------------------- closed forms

@pytest.mark.parametrize("k", ["1024", "2048"])
def test_closed_forms_real_keys(k):
    p, q = KEYS[k]
    n = p * q
    n2 = n * n
    rng = random.Random(int(k))
    for _ in range(3):
        m = rng.randrange(n)
        # Enc(m; r = 1) = (1 + n)^m = 1 + m n mod n^2 (binomial theorem; g = n + 1)
        assert paillier.encrypt(n, m, 1) == (1 + m * n) % n2
        r = rng.randrange(1, n)
        # Enc(0; r) is an n-th power residue: its n-th-root structure means Dec = 0
        assert paillier.decrypt(p, q, paillier.encrypt(n, 0, r)) == 0
        # r^n mod n^2 depends only on r mod n (reading c3)
        assert paillier.encrypt(n, m, r) == paillier.encrypt(n, m, r + 3 * n)


def test_mu_closed_form():
    """With g = n+1: L(g^lam mod n^2) = lam mod n, so mu = lam^-1 mod n (reading c1)."""
    p, q = KEYS["1024"]
    n = p * q
    lam = math.lcm(p - 1, q - 1)
    assert paillier.L(pow(n + 1, lam, n * n), n) == lam % n


def _crt_decrypt(p, q, c):
    # an independent second algorithm (CRT, Paillier'99 §7), used only to cross-check Eq. 4
    hp = pow(-q % p, -1, p)
    hq = pow(-p % q, -1, q)
    mp = (pow(c, p - 1, p * p) - 1) // p * hp % p
    mq = (pow(c, q - 1, q * q) - 1) // q * hq % q
    return mq + q * ((mp - mq) * pow(q, -1, p) % p)


@pytest.mark.parametrize("k", ["1024", "2048"])
def test_decrypt_matches_crt_algorithm(k):
    p, q = KEYS[k]
    n = p * q
    rng = random.Random(5)
    for _ in range(3):
        m = rng.randrange(n)
        c = paillier.encrypt(n, m, rng.randrange(1, n))
        assert paillier.decrypt(p, q, c) == m == _crt_decrypt(p, q, c)


@pytest.mark.parametrize("k", ["1024"])
def test_homomorphic_invariants_real_key(k):
    p, q = KEYS[k]
    n = p * q
    rng = random.Random(11)
    a, b, e = rng.randrange(n), rng.randrange(n), rng.randrange(1 << 32)
    ca = paillier.encrypt(n, a, rng.randrange(1, n))
    cb = paillier.encrypt(n, b, rng.randrange(1, n))
    assert paillier.decrypt(p, q, paillier.add(n, ca, cb)) == (a + b) % n
    assert paillier.decrypt(p, q, paillier.scalar_mul(n, ca, e)) == a * e % n
    assert paillier.scalar_mul(n, ca, 0) == 1
    assert paillier.scalar_mul(n, ca, 1) == ca


def test_reduce_segments_sum_permutation_and_empty():
    p, q = KEYS["toy16"]
    n = p * q
    rng = random.Random(3)
    ms = [rng.randrange(n) for _ in range(40)]
    cs = [paillier.encrypt(n, m, rng.randrange(1, n)) for m in ms]
    offsets = [0, 5, 5, 17, 40]  # includes an empty segment
    out = paillier.reduce_segments(n, cs, offsets)
    assert out[1] == 1  # empty product = 1 = Enc(0; r = 1)
    for j in range(4):
        assert paillier.decrypt(p, q, out[j]) == sum(ms[offsets[j]:offsets[j + 1]]) % n
    perm = list(range(40))
    rng.shuffle(perm)
    inv = {v: i for i, v in enumerate(perm)}
    cs_perm = [cs[perm[t]] for t in range(40)]
    idx = [inv[t] for t in range(40)]
    assert paillier.reduce_segments(n, cs_perm, offsets, idx) == out


# ----------------------------------------------------------------------------- Montgomery

@pytest.mark.parametrize("limbs", [2, 32, 64])
def test_mont_mul_definition(limbs):
    rng = random.Random(limbs)
    R = 1 << (32 * limbs)
    for _ in range(20):
        N = rng.randrange(3, R) | 1
        a, b = rng.randrange(N), rng.randrange(N)
        z = montgomery.mont_mul(a, b, N, limbs)
        assert 0 <= z < N and (z * R - a * b) % N == 0
        # mont(a R mod N, 1) = a
        assert montgomery.mont_mul(a * R % N, 1, N, limbs) == a


# ----------------------------------------------------------------------------- limbs / r

def test_limb_roundtrip():
    rng = random.Random(0)
    for w in (1, 4, 64):
        x = rng.getrandbits(32 * w)
        assert paillier.from_limbs(paillier.to_limbs(x, w)) == x


def test_draw_r_range_and_determinism():
    p, q = KEYS["2048"]
    n = p * q
    for i in range(5):
        r = philox.draw_r(n, 1234, i, 64)
        assert 1 <= r < (1 << (n.bit_length() - 1)) <= n
        assert r == philox.draw_r(n, 1234, i, 64)
    assert philox.draw_r(n, 1234, 0, 64) != philox.draw_r(n, 1234, 1, 64)
    # toy key: bits(n) - 1 = 15 bits of randomness
    ptoy, qtoy = KEYS["toy16"]
    for i in range(50):
        assert 1 <= philox.draw_r(ptoy * qtoy, 9, i, 32) < (1 << 15)


def test_miller_rabin_with_given_bases():
    # primes pass every base; composites are caught by some base; base 2 alone is fooled by the
    # strong pseudoprime 2047 = 23 * 89 (a textbook fact), bases 2 and 3 by 1373653 = 829 * 1657
    for pr in (3, 5, 7, 101, 7919, (1 << 61) - 1, (1 << 89) - 1):
        assert paillier.miller_rabin_bases(pr, [b for b in (2, 3, 5, 7, 11) if b < pr - 1] + [pr - 1])
    assert paillier.miller_rabin_bases(2047, [2]) and not paillier.miller_rabin_bases(2047, [3])
    assert paillier.miller_rabin_bases(1373653, [2, 3]) and not paillier.miller_rabin_bases(1373653, [5])
    for c in (561, 1105, 1729, 2465, 2821, 6601, 8911):  # Carmichael numbers: base 2 catches them
        assert not paillier.miller_rabin_bases(c, [2])
    rng = random.Random(8)
    for _ in range(300):  # agreement with trial division on random odd 20-bit numbers, 8 random bases
        x = rng.randrange(3, 1 << 20) | 1
        is_p = all(x % d for d in range(3, int(math.isqrt(x)) + 1, 2))
        assert paillier.miller_rabin_bases(x, [rng.randrange(2, x - 1) for _ in range(8)]) == is_p

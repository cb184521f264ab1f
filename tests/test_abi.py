"""CPU tests of the C ABI: the library loads, exports every symbol include/flb_paillier.h declares,
and its host-side logic (key import/generation/export, argument validation, cost accounting)
behaves — no device work is launched here."""

import ctypes
import os
import re
import subprocess

import pytest

import paper_conf_icde_zeng0fcpcwg23_b200 as flb
from paper_conf_icde_zeng0fcpcwg23_b200 import _lib
from tests.helpers import golden_keys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "flb_paillier.h")
KEYS = golden_keys()


def declared_symbols():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(flb_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    syms = declared_symbols()
    for s in ["flb_keygen", "flb_key_from_primes", "flb_encrypt", "flb_decrypt", "flb_add", "flb_scalar_mul",
              "flb_reduce_segments", "flb_pack", "flb_unpack", "flb_unpack_sums", "flb_last_error"]:
        assert s in syms


def test_library_exports_every_declared_symbol():
    out = subprocess.run(["nm", "-D", "--defined-only", _lib.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (flb_[a-z0-9_]+)\b", out))
    missing = [s for s in declared_symbols() if s not in exported]
    assert not missing, missing
    # and the binding binds exactly the declared set
    assert sorted(_lib.SIGNATURES) == declared_symbols()
    lib = ctypes.CDLL(_lib.LIB_PATH)
    for s in declared_symbols():
        getattr(lib, s)


def test_library_is_sm100a():
    out = subprocess.run(["cuobjdump", "--list-elf", _lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


@pytest.mark.parametrize("name,bits,ptw,ctw", [("toy9", 9, 32, 64), ("toy16", 16, 32, 64), ("1024", 1024, 32, 64),
                                               ("2048", 2048, 64, 128), ("3072", 3072, 96, 192),
                                               ("4096", 4096, 128, 256)])
def test_key_import_export(name, bits, ptw, ctw):
    p, q = KEYS[name]
    pub, priv = flb.key_from_primes(q, p)  # order does not matter; p becomes the larger
    assert (pub.bits, pub.pt_words, pub.ct_words) == (bits, ptw, ctw)
    P, Q, N = priv.export()
    assert (P, Q, N) == (max(p, q), min(p, q), p * q)
    assert pub.slot_capacity(32) == (bits - 1) // 32


def test_keygen_deterministic_and_valid():
    pub, priv = flb.keygen(1024, 12345)
    p, q, n = priv.export()
    pub2, priv2 = flb.keygen(1024, 12345)
    assert priv2.export() == (p, q, n)
    assert flb.keygen(1024, 12346)[1].export() != (p, q, n)
    assert n.bit_length() == 1024 and p.bit_length() == q.bit_length() == 512
    for x in (p, q):  # independent check: Fermat + small trial division
        assert all(pow(b, x - 1, x) == 1 for b in (2, 3, 5, 7, 11))
        assert all(x % d for d in range(3, 2000, 2))


@pytest.mark.parametrize("p,q,code", [(251, 251, -4), (251, 255, -4), (250, 241, -4), (1, 241, -4),
                                      (7, 3, -4)])  # gcd(21, 12) = 3
def test_key_import_rejects(p, q, code):
    with pytest.raises(flb.FlbError) as e:
        flb.key_from_primes(p, q)
    assert e.value.code == code


def test_key_import_rejects_oversize():
    p = (1 << 2100) + 1  # size check happens before primality
    with pytest.raises(flb.FlbError) as e:
        flb.key_from_primes(p, p + 2)
    assert e.value.code == -5


def test_keygen_rejects_bad_size():
    with pytest.raises(flb.FlbError) as e:
        flb.keygen(1000, 1)
    assert e.value.code == -1


def test_batch_calls_validate_before_launch():
    p, q = KEYS["1024"]
    pub, priv = flb.key_from_primes(p, q)
    L = _lib.LIB
    assert L.flb_encrypt(pub.handle, None, None, 0, 0, None, 4, None) == -1
    assert L.flb_decrypt(priv.handle, None, None, 4, None) == -1
    assert L.flb_add(pub.handle, None, None, None, 4, None) == -1
    assert L.flb_scalar_mul(pub.handle, 16, 16, 0, 16, 4, None) == -1  # e_words = 0
    assert L.flb_reduce_segments(pub.handle, None, 3, None, 3, None, 2, 0, None, None) == -1
    assert "null" in L.flb_last_error().decode()
    assert L.flb_reduce_segments(pub.handle, 16, 3, None, 4, 16, 2, 0, 16, None) == -1  # entries > inputs, no idx
    # count = 0 is a no-op that needs no device
    assert L.flb_encrypt(pub.handle, 16, None, 0, 0, 16, 0, None) == 0
    bad = [(1.0, 29, 3, 32, 32), (1.0, 29, 4, 33, 1), (0.0, 29, 3, 32, 1), (1.0, 53, 11, 64, 1), (1.0, 29, 3, 32, 0)]
    for a, qb, pb, sb, sl in bad:
        cs = _lib.CodecStruct(a, qb, pb, sb, sl)
        assert L.flb_pack(pub.handle, ctypes.byref(cs), 16, 10, 16, None) == -1
        assert L.flb_unpack(pub.handle, ctypes.byref(cs), 16, 10, None, 1, 16, None) == -1
    # b = pad_bits overflow bits hold at most 2^b summands per slot
    cs = _lib.CodecStruct(1.0, 29, 3, 32, 31)
    assert L.flb_unpack(pub.handle, ctypes.byref(cs), 16, 10, None, 9, 16, None) == -1
    assert "2^pad_bits" in L.flb_last_error().decode()
    assert L.flb_unpack(pub.handle, ctypes.byref(cs), 16, 0, None, 8, 16, None) == 0  # 8 = 2^3 is allowed


def _sliding_mults(e, w):
    """Independent count of a left-to-right odd-power sliding window (table + squarings + products)."""
    bits = bin(e)[2:]
    table = 1 << (w - 1)
    cost = table if table > 1 else 0
    i, first = 0, True
    while i < len(bits):
        if bits[i] == "0":
            cost += 1
            i += 1
            continue
        j = min(len(bits), i + w)
        while bits[j - 1] == "0":
            j -= 1
        cost += 0 if first else (j - i) + 1
        first = False
        i = j
    return cost


def test_op_cost_matches_independent_window_count():
    p, q = KEYS["2048"]
    pub, priv = flb.key_from_primes(p, q)
    n = p * q
    mm, lp = flb.op_cost(pub, "encrypt")
    best = min(_sliding_mults(n, w) for w in range(1, 8))
    assert mm == best + 3  # + to-Montgomery, m*n, final product
    assert lp == mm * (2 * 128 * 128 + 128)
    mm_d, lp_d = flb.op_cost(priv, "decrypt")
    bd = sum(min(_sliding_mults(P - 1, w) for w in range(1, 8)) for P in (p, q))
    assert mm_d == bd + 2 * 4 + 2
    assert flb.op_cost(pub, "add") == (2, 2 * (2 * 128 * 128 + 128))


def test_mod_create_and_rsa_keygen_host_logic():
    for bits, words in [(61, 32), (1024, 32), (1025, 64), (2048, 64), (3000, 96), (4096, 128), (8192, 256)]:
        n = (1 << (bits - 1)) | 1
        assert flb.Modulus(n).words == words
    for bad in (0, 1, 2, 10, 1 << 8192):
        with pytest.raises(flb.FlbError):
            flb.Modulus(bad)
    n, e, d, p, q = flb.rsa_keygen(512, 7)
    assert p > q and p * q == n and n.bit_length() == 512 and e == 65537
    assert (e * d) % ((p - 1) * (q - 1)) == 1
    assert all(pow(b, x - 1, x) == 1 for x in (p, q) for b in (2, 3, 5))
    assert flb.rsa_keygen(512, 7) == (n, e, d, p, q)
    with pytest.raises(flb.FlbError):
        flb.rsa_keygen(100, 1)


def _sliding_counts(e, w):
    """(multiplications, of which squarings) of the odd-power sliding window, counted independently."""
    bits = bin(e)[2:]
    table = 1 << (w - 1)
    mults, sq = (table, 1) if table > 1 else (0, 0)
    i, first = 0, True
    while i < len(bits):
        if bits[i] == "0":
            mults, sq, i = mults + 1, sq + 1, i + 1
            continue
        j = min(len(bits), i + w)
        while bits[j - 1] == "0":
            j -= 1
        if not first:
            mults, sq = mults + (j - i) + 1, sq + (j - i)
        first = False
        i = j
    return mults, sq


def test_op_cost_tensor_core_paths():
    """Accounting of the tensor-core kernels (bench.py's roofline): Montgomery products per element,
    IMAD-pipe limb products (S^2 per product; block squaring with triangular diagonal blocks:
    4 x (X (X + 1) / 2 + 1.5 X^2) at S = 64 (X = 16 limbs per lane), 2 x (X (X + 1) / 2 + X^2 / 2)
    at S = 32) and the u8 MACs the triangular Toeplitz MMAs issue, against an independent window count."""
    p, q = KEYS["2048"]
    pub, priv = flb.key_from_primes(p, q)
    sp, h = 64, 32

    def best(e):
        costs = [_sliding_counts(e, w) for w in range(1, 8)]
        m = min(c[0] for c in costs)
        return m, {c[1] for c in costs if c[0] == m}

    mm, lp = flb.op_cost(priv, "decrypt_tc")
    (mp, sqp), (mq, sqq) = best(p - 1), best(q - 1)
    assert mm == mp + mq + 2 * 3
    X = 16  # limbs per lane at both frames
    sq64 = 4 * (X * (X + 1) // 2 + X * X + X * X // 2)   # diagonal, full and half off-diagonal blocks
    sq32 = 2 * (X * (X + 1) // 2 + X * X // 2)           # diagonal, half cross block
    assert any(lp == (mm - a - b) * sp * sp + (a + b) * sq64 for a in sqp for b in sqq)
    def macs(S):
        # (K, column) pairs the triangular K-slices cover: q = t N' mod R reaches column j from
        # K <= j; the high half of q N (columns KB-8+j) from K >= j - 39 within the slice's 32 rows
        KB = 4 * S
        lo = sum(32 * (KB - 32 * ks) for ks in range(KB // 32))
        hi = sum(32 * min(KB, 32 * ks + 48) for ks in range(KB // 32))
        assert lo < KB * KB and hi < KB * KB
        return lo + hi

    assert flb.op_cost(priv, "decrypt_tc_macs") == (mm, mm * macs(sp))
    mm_e, lp_e = flb.op_cost(priv, "encrypt_crt_tc")
    (ep, esp), (eq, esq) = best(p), best(q)
    s1 = (2 + eq + 1) + (2 + ep + 1)      # stage 1: r^Q mod p, r^P mod q at the half frame
    s2 = (1 + ep + 2) + (1 + eq + 2)      # stage 2: y^P mod P^2
    assert mm_e == s1 + s2
    # stage 1 (h = 32 words, two lanes), stage 2 (64 words, four lanes)
    assert any(lp_e == (s1 - a - b) * h * h + (a + b) * sq32
               + (s2 - a - b) * sp * sp + (a + b) * sq64 for a in esp for b in esq)
    assert flb.op_cost(priv, "encrypt_crt_tc_macs") == (mm_e, s1 * macs(h) + s2 * macs(sp))
    # 1024-bit keys have no two-stage (half-frame) path: one stage per prime, (1 + m n) r^n mod P^2 with
    # the exponent n in the 32-word frame (entry, table + schedule of n, m n, final product)
    p1, q1 = KEYS["1024"]
    _, priv1 = flb.key_from_primes(p1, q1)
    mm1, lp1 = flb.op_cost(priv1, "encrypt_crt_tc")
    (mn, sqn) = best(p1 * q1)
    assert mm1 == 2 * (1 + mn + 2)
    sq32 = 2 * (X * (X + 1) // 2 + X * X // 2)
    assert any(lp1 == (mm1 - 2 * a) * 32 * 32 + 2 * a * sq32 for a in sqn)
    assert flb.op_cost(priv1, "encrypt_crt_tc_macs") == (mm1, mm1 * macs(32))

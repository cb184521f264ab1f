"""GPU parity: every CUDA entry point against the oracle, bit-exact.

Inputs are seeded (synthetic/), expected values come only from oracle/; the CUDA path is called
through the C ABI via the thin Python binding.  Sizes span several warps/blocks with ragged tails
and stay small enough for the pure-Python oracle.
"""

import random

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover - CPU container
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402
from oracle import montgomery, paillier, philox  # noqa: E402
from tests.helpers import from_dev, golden_keys, to_dev  # noqa: E402

pytestmark = pytest.mark.gpu

KEYS = golden_keys()
_CACHE = {}


def key(name):
    if name not in _CACHE:
        p, q = KEYS[name]
        _CACHE[name] = flb.key_from_primes(p, q) + (p, q)
    return _CACHE[name]


# number of elements per key size: several warps plus a ragged tail, oracle cost bounded
COUNT = {"toy9": 200, "toy16": 150, "1024": 67, "2048": 21, "3072": 5, "4096": 3}
ALL = ["toy9", "toy16", "1024", "2048", "3072", "4096"]


def rand_below(bound, count, seed):
    return synthetic.uniform_below(bound, count, seed)


def _unit(rng, n):
    """r in Z*_n: decryption is only defined for ciphertexts that are units."""
    import math
    while True:
        r = rng.randrange(1, n)
        if math.gcd(r, n) == 1:
            return r


# ----------------------------------------------------------------------------- Montgomery primitive

@pytest.mark.parametrize("name", ALL)
def test_mont_mul(name):
    pub, priv, p, q = key(name)
    n2 = (p * q) ** 2
    cnt = 100
    a = rand_below(n2, cnt, 1)
    b = rand_below(n2, cnt, 2)
    R = 1 << (32 * pub.ct_words)
    # edge operands: 0, 1, N-1, R mod N, and (N-1)^2
    a[:5] = [0, 1, n2 - 1, R % n2, n2 - 1]
    b[:5] = [n2 - 1, n2 - 1, n2 - 1, R % n2, n2 - 1]
    out = flb.debug_mont_mul(pub, to_dev(a, pub.ct_words), to_dev(b, pub.ct_words))
    got = from_dev(out)
    for i in range(cnt):
        assert got[i] == montgomery.mont_mul(a[i], b[i], n2, pub.ct_words), i


# ----------------------------------------------------------------------------- encrypt

@pytest.mark.parametrize("name", ALL)
def test_encrypt_caller_r(name):
    pub, priv, p, q = key(name)
    n = p * q
    cnt = COUNT[name]
    m = rand_below(n, cnt, 11)
    r = [x if x else 1 for x in rand_below(n, cnt, 12)]  # any r: Eq. 3 is defined for all r
    m[0], m[-1] = 0, n - 1
    c = flb.encrypt(pub, to_dev(m, pub.pt_words), r=to_dev(r, pub.pt_words))
    got = from_dev(c)
    for i in range(cnt):
        assert got[i] == paillier.encrypt(n, m[i], r[i]), i


@pytest.mark.parametrize("name", ALL)
def test_encrypt_philox_r(name):
    pub, priv, p, q = key(name)
    n = p * q
    cnt = COUNT[name]
    m = rand_below(n, cnt, 13)
    seed, ctr0 = 0x0123456789ABCDEF, 1000
    c = flb.encrypt(pub, to_dev(m, pub.pt_words), seed=seed, ctr0=ctr0)
    got = from_dev(c)
    for i in range(cnt):
        r = philox.draw_r(n, seed, ctr0 + i, pub.pt_words)
        assert got[i] == paillier.encrypt(n, m[i], r), i


@pytest.mark.parametrize("name", ALL)
def test_encrypt_crt_matches_oracle(name):
    """Key-holder CRT encryption gives exactly Eq. 3's value, for caller and Philox r (any r)."""
    pub, priv, p, q = key(name)
    n = p * q
    cnt = COUNT[name]
    m = rand_below(n, cnt, 14)
    r = [x if x else 1 for x in rand_below(n, cnt, 15)]
    m[0], m[-1] = 0, n - 1
    r[1] = p if p < n else 1          # r sharing a factor with n: still the public-path value
    got = from_dev(flb.encrypt_crt(priv, to_dev(m, pub.pt_words), r=to_dev(r, pub.pt_words)))
    for i in range(cnt):
        assert got[i] == paillier.encrypt(n, m[i], r[i]), i
    seed, ctr0 = 0xFEDCBA9876543210, 77
    got = from_dev(flb.encrypt_crt(priv, to_dev(m, pub.pt_words), seed=seed, ctr0=ctr0))
    for i in range(cnt):
        assert got[i] == paillier.encrypt(n, m[i], philox.draw_r(n, seed, ctr0 + i, pub.pt_words)), i


def test_encrypt_crt_equals_public_path_at_scale():
    pub, priv, p, q = key("2048")
    n = p * q
    M = 3000
    m = to_dev(rand_below(n, M, 16), pub.pt_words)
    a = flb.encrypt(pub, m, seed=5, ctr0=9)
    b = flb.encrypt_crt(priv, m, seed=5, ctr0=9)
    assert torch.equal(a, b)
    got = from_dev(b)
    for i in (0, 1, 1234, M - 1):
        assert got[i] == paillier.encrypt(n, from_dev(m[i:i + 1])[0], philox.draw_r(n, 5, 9 + i, pub.pt_words))


# ----------------------------------------------------------------------------- decrypt

@pytest.mark.parametrize("name", ALL)
def test_decrypt(name):
    pub, priv, p, q = key(name)
    n = p * q
    cnt = COUNT[name]
    rng = random.Random(21)
    m = rand_below(n, cnt, 22)
    m[0], m[-1] = 0, n - 1
    cs = [paillier.encrypt(n, m[i], _unit(rng, n)) for i in range(cnt)]
    got = from_dev(flb.decrypt(priv, to_dev(cs, pub.ct_words)))
    for i in range(cnt):
        assert got[i] == paillier.decrypt(p, q, cs[i]) == m[i], i


@pytest.mark.parametrize("name", ["toy9", "toy16"])
def test_decrypt_arbitrary_residues(name):
    """Every unit c < n^2 is a ciphertext (Paillier's bijection Z_n x Z*_n -> Z*_{n^2}): CRT = Eq. 4."""
    pub, priv, p, q = key(name)
    n2 = (p * q) ** 2
    cs = rand_below(n2, 300, 23)
    got = from_dev(flb.decrypt(priv, to_dev(cs, pub.ct_words)))
    import math
    for i, c in enumerate(cs):
        if math.gcd(c, p * q) == 1:
            assert got[i] == paillier.decrypt(p, q, c), i


def test_toy9_exhaustive_roundtrip():
    pub, priv, p, q = key("toy9")
    n = p * q
    m = list(range(n))
    import math
    c = flb.encrypt(pub, to_dev(m, pub.pt_words), seed=99)
    got = from_dev(flb.decrypt(priv, c))
    cc = from_dev(c)
    units = 0
    for i in range(n):
        r = philox.draw_r(n, 99, i, pub.pt_words)
        assert cc[i] == paillier.encrypt(n, i, r), i
        if math.gcd(r, n) == 1:  # Philox r sharing a factor with a toy n is not a valid r (L90)
            units += 1
            assert got[i] == i, i
    assert units > 250


# ----------------------------------------------------------------------------- add / scalar mul

@pytest.mark.parametrize("name", ALL)
def test_add(name):
    pub, priv, p, q = key(name)
    n2 = (p * q) ** 2
    cnt = 3 * COUNT[name] + 5
    a = rand_below(n2, cnt, 31)
    b = rand_below(n2, cnt, 32)
    a[0], b[0] = n2 - 1, n2 - 1
    a[1], b[1] = 0, 5
    out = flb.add(pub, to_dev(a, pub.ct_words), to_dev(b, pub.ct_words))
    got = from_dev(out)
    for i in range(cnt):
        assert got[i] == paillier.add(p * q, a[i], b[i]), i


def test_add_aliasing():
    pub, priv, p, q = key("1024")
    n2 = (p * q) ** 2
    a = rand_below(n2, 50, 33)
    b = rand_below(n2, 50, 34)
    ta, tb = to_dev(a, pub.ct_words), to_dev(b, pub.ct_words)
    flb.add(pub, ta, tb, out=ta)
    assert from_dev(ta) == [x * y % n2 for x, y in zip(a, b)]


@pytest.mark.parametrize("name", ALL)
@pytest.mark.parametrize("e_words", [1, 2, 5])
def test_scalar_mul(name, e_words):
    pub, priv, p, q = key(name)
    n2 = (p * q) ** 2
    cnt = COUNT[name] + 3
    c = rand_below(n2, cnt, 41)
    rng = random.Random(42 + e_words)
    e = [rng.getrandbits(32 * e_words) >> rng.randrange(0, 32 * e_words) for _ in range(cnt)]
    e[0], e[1], e[2] = 0, 1, (1 << (32 * e_words)) - 1
    et = torch.from_numpy(synthetic.ints_to_limbs(e, e_words).view(np.int32)).cuda()
    got = from_dev(flb.scalar_mul(pub, to_dev(c, pub.ct_words), et))
    for i in range(cnt):
        assert got[i] == paillier.scalar_mul(p * q, c[i], e[i]), i


# ----------------------------------------------------------------------------- reduce

def _check_reduce(name, cnt, offsets, idx=None, hint=0):
    pub, priv, p, q = key(name)
    n2 = (p * q) ** 2
    cs = rand_below(n2, cnt, 51)
    off = torch.tensor(offsets, dtype=torch.int64).cuda()
    it = None if idx is None else torch.tensor(idx, dtype=torch.int64).cuda()
    got = from_dev(flb.reduce_segments(pub, to_dev(cs, pub.ct_words), off, idx=it, max_segment_len=hint))
    exp = paillier.reduce_segments(p * q, cs, offsets, idx)
    assert got == exp


@pytest.mark.parametrize("name", ["toy16", "1024", "2048"])
def test_reduce_ragged_with_empty(name):
    offs = synthetic.random_segments(300, 37, seed=5).tolist()
    _check_reduce(name, 300, offs)


def test_reduce_gather_and_permutation():
    rng = random.Random(6)
    idx = list(range(200))
    rng.shuffle(idx)
    offs = [0, 1, 1, 64, 65, 129, 200]
    _check_reduce("1024", 200, offs, idx)


@pytest.mark.parametrize("hint", [0, 700])
def test_reduce_long_segment_multilevel(hint):
    # one segment of 700 (> 64^1: two levels), one of 3, one empty
    _check_reduce("1024", 703, [0, 700, 703, 703], None, hint)


def test_reduce_all_empty():
    pub, priv, p, q = key("1024")
    off = torch.zeros(5, dtype=torch.int64).cuda()
    c = torch.zeros((0, pub.ct_words), dtype=torch.int32).cuda()
    got = from_dev(flb.reduce_segments(pub, c, off))
    assert got == [1, 1, 1, 1]


# ----------------------------------------------------------------------------- homomorphic invariants at scale

def test_invariants_at_scale_2048():
    """Dec(Enc(a) Enc(b)) = a + b and Dec(Enc(a)^e) = e a mod n over a large batch (GPU only)."""
    pub, priv, p, q = key("2048")
    n = p * q
    M = 4096
    a = rand_below(n // 2, M, 61)
    b = rand_below(n // 2, M, 62)
    ca = flb.encrypt(pub, to_dev(a, pub.pt_words), seed=1)
    cb = flb.encrypt(pub, to_dev(b, pub.pt_words), seed=2, ctr0=M)
    s = from_dev(flb.decrypt(priv, flb.add(pub, ca, cb)))
    assert s == [x + y for x, y in zip(a, b)]
    e = torch.randint(0, 2 ** 31, (M, 1), dtype=torch.int32, generator=torch.Generator().manual_seed(3)).cuda()
    sm = from_dev(flb.decrypt(priv, flb.scalar_mul(pub, ca, e)))
    ev = e.cpu().numpy().ravel().tolist()
    assert sm == [x * y % n for x, y in zip(a, ev)]

"""Tensor-core Montgomery path in the wide frames (csrc/flb_tc.cuh at S = 128: KB = 512 byte
columns, two 256-column MMAs per Toeplitz K-slice, all 512 TMEM columns, one CTA per SM, 8 lanes per
element in the product phase) and the public-key encryption on the tensor cores (n^2 of 64 or 128
words, Eq. 3): bit-exact against the CUDA-core CIOS kernels (FLB_TC=0) and against the
oracle on sampled elements, on ragged tile counts and edge operands."""

import os

import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402
from oracle import paillier, philox  # noqa: E402
from tests.helpers import from_dev, golden_keys, to_dev  # noqa: E402

pytestmark = pytest.mark.gpu
KEYS = golden_keys()


def _env(fn, tc):
    """FLB_TC = "0": CIOS kernels; "1": automatic (public-key encryption on the tensor cores from 96
    elements per SM); "2": the tensor-core kernels at every batch size."""
    old = os.environ.get("FLB_TC")
    try:
        os.environ["FLB_TC"] = tc
        out = fn()
        torch.cuda.synchronize()
        return out
    finally:
        if old is None:
            os.environ.pop("FLB_TC", None)
        else:
            os.environ["FLB_TC"] = old


@pytest.fixture(scope="module", params=["1024", "2048"])
def key(request):
    p, q = KEYS[request.param]
    return flb.key_from_primes(p, q) + (p, q)


@pytest.mark.parametrize("count", [1, 129, 300])
def test_public_encrypt_tc_matches_cios_and_oracle(key, count):
    pub, priv, p, q = key
    n = p * q
    m_int = synthetic.uniform_below(n, count, 1100 + count)
    m_int[0] = 0
    if count > 1:
        m_int[1] = n - 1
    m = to_dev(m_int, pub.pt_words)
    seed, ctr0 = 0x9B000000 + count, 5
    tc = _env(lambda: flb.encrypt(pub, m, seed=seed, ctr0=ctr0), "2")
    cios = _env(lambda: flb.encrypt(pub, m, seed=seed, ctr0=ctr0), "0")
    assert torch.equal(tc, cios)
    got = from_dev(tc)
    for i in sorted({0, count // 2, count - 1}):
        assert got[i] == paillier.encrypt(n, m_int[i], philox.draw_r(n, seed, ctr0 + i, pub.pt_words)), i
    # and it decrypts
    assert from_dev(flb.decrypt(priv, tc)) == m_int


@pytest.mark.parametrize("extra", [1, 64, 100, 128 * 5 + 3])
def test_public_encrypt_tc_half_units(key, extra):
    """Batches one round of the persistent grid plus a few tiles: the last, incomplete round runs as half
    units (64 elements on the rows of product pass 0, one pass) — including an empty second half and a
    ragged first half; bit-exact against CIOS."""
    pub, priv, p, q = key
    n = p * q
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    per_sm = 1 if pub.ct_words >= 96 else 2  # k_tc_exp CTAs per SM (flb_tc.cuh Cfg::CTAS_PER_SM)
    count = sms * per_sm * 128 + extra
    m = to_dev(synthetic.uniform_below(n, count, 1150 + extra), pub.pt_words)
    tc = _env(lambda: flb.encrypt(pub, m, seed=0x4A11, ctr0=2), "2")
    cios = _env(lambda: flb.encrypt(pub, m, seed=0x4A11, ctr0=2), "0")
    bad = (tc != cios).any(dim=1).nonzero().flatten().tolist()
    assert not bad, (len(bad), bad[:5])


def test_public_encrypt_tc_caller_r_edge(key):
    """caller-supplied r: r = 1 (Enc(m; 1) = 1 + m n), r = n - 1, r = p (not a unit: the function is still
    defined as the integer formula)."""
    pub, priv, p, q = key
    n = p * q
    rs = [1, n - 1, p, 2, n - 2] + synthetic.uniform_below(n, 3, 1200)
    ms = synthetic.uniform_below(n, len(rs), 1201)
    r = to_dev(rs, pub.pt_words)
    m = to_dev(ms, pub.pt_words)
    tc = from_dev(_env(lambda: flb.encrypt(pub, m, r=r), "2"))
    for i in range(len(rs)):
        assert tc[i] == paillier.encrypt(n, ms[i], rs[i]), i


@pytest.fixture(scope="module", params=["3072", "4096"])
def k4096(request):
    p, q = KEYS[request.param]
    return flb.key_from_primes(p, q) + (p, q)


@pytest.mark.parametrize("count", [1, 130])
def test_decrypt_4096_tc_matches_cios_and_oracle(k4096, count):
    """3072/4096-bit decryption: c^(P-1) mod P^2 with P^2 of 96 / 128 words on the S = 96 / 128 kernel
    (S = 96: eight lanes of 12 limbs, KB = 384 byte columns in a 256 + 128-column MMA pair)."""
    pub, priv, p, q = k4096
    n = p * q
    m_int = synthetic.uniform_below(n, count, 1300 + count)
    c = _env(lambda: flb.encrypt_crt(priv, to_dev(m_int, pub.pt_words), seed=17), "0")
    tc = _env(lambda: flb.decrypt(priv, c), "1")
    cios = _env(lambda: flb.decrypt(priv, c), "0")
    assert torch.equal(tc, cios)
    assert from_dev(tc) == m_int
    cs = from_dev(c)
    for i in sorted({0, count - 1}):
        assert paillier.decrypt(p, q, cs[i]) == m_int[i]


@pytest.mark.parametrize("count", [1, 130])
def test_keyholder_encrypt_4096_tc_matches_cios_and_oracle(k4096, count):
    """3072/4096-bit key-holder encryption: stage 1 at H = 64 and stage 2 (1 + m n) y^P mod P^2 at
    S = 96 / 128 on the tensor cores, same bits as the CIOS kernels and the oracle's Eq. 3."""
    pub, priv, p, q = k4096
    n = p * q
    m_int = synthetic.uniform_below(n, count, 1400 + count)
    m = to_dev(m_int, pub.pt_words)
    tc = _env(lambda: flb.encrypt_crt(priv, m, seed=23, ctr0=1), "1")
    cios = _env(lambda: flb.encrypt_crt(priv, m, seed=23, ctr0=1), "0")
    assert torch.equal(tc, cios)
    got = from_dev(tc)
    i = count - 1
    assert got[i] == paillier.encrypt(n, m_int[i], philox.draw_r(n, 23, 1 + i, pub.pt_words))


def test_tc_product_phase_128():
    """The S = 128 product phase (8 lanes, general row scan also for squarings): exact 256-limb products."""
    words, count = 128, 128
    a_int = synthetic.uniform_below(1 << (32 * words), count, 1500)
    b_int = synthetic.uniform_below(1 << (32 * words), count, 1501)
    top = (1 << (32 * words)) - 1
    a_int[:3] = [top, 0, 1 << (32 * words - 1)]
    b_int[:3] = [top, top, top]
    a, b = to_dev(a_int, words), to_dev(b_int, words)
    t = from_dev(flb.debug_tc_product(a, b, square=False))
    t2 = from_dev(flb.debug_tc_product(a, a, square=True))
    for i in range(count):
        assert t[i] == a_int[i] * b_int[i], i
        assert t2[i] == a_int[i] * a_int[i], i


@pytest.mark.parametrize("count", [1, 129, 300, 20000])
def test_keyholder_encrypt_1024_one_stage_tc(count):
    """1024-bit key-holder encryption (no half frame): (1 + m n) r^n mod P^2 for both primes on the S = 32
    tensor-core kernel (exponent n), then the CRT recombination; same bits as the CIOS k_encrypt_crt and
    as the oracle's Eq. 3 (20,000 elements: the automatic dispatch takes the tensor cores too)."""
    p, q = KEYS["1024"]
    pub, priv = flb.key_from_primes(p, q)
    n = p * q
    m_int = synthetic.uniform_below(n, count, 1600 + count)
    m_int[0] = 0
    if count > 1:
        m_int[-1] = n - 1
    m = to_dev(m_int, pub.pt_words)
    tc = _env(lambda: flb.encrypt_crt(priv, m, seed=31, ctr0=4), "2")
    cios = _env(lambda: flb.encrypt_crt(priv, m, seed=31, ctr0=4), "0")
    assert torch.equal(tc, cios)
    if count >= 20000:
        auto = _env(lambda: flb.encrypt_crt(priv, m, seed=31, ctr0=4), "1")
        assert torch.equal(auto, cios)
    got = from_dev(tc)
    for i in sorted({0, count // 2, count - 1}):
        assert got[i] == paillier.encrypt(n, m_int[i], philox.draw_r(n, 31, 4 + i, pub.pt_words)), i

"""Tensor-core Montgomery path (csrc/flb_tc.cuh, the default key-holder stage 2 at 2048 bits):
bit-exact against the oracle and against the CIOS kernel (FLB_TC=0) on ragged tile counts and on
edge-case operands (m = 0, m = n - 1, r = 1, r = n - 1, r a multiple of p or q)."""

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


@pytest.fixture(scope="module")
def k2048():
    p, q = KEYS["2048"]
    return flb.key_from_primes(p, q) + (p, q)


def _both(priv, m, **kw):
    old = os.environ.get("FLB_TC")
    try:
        os.environ["FLB_TC"] = "0"
        cios = flb.encrypt_crt(priv, m, **kw)
        os.environ["FLB_TC"] = "1"
        tc = flb.encrypt_crt(priv, m, **kw)
    finally:
        if old is None:
            os.environ.pop("FLB_TC", None)
        else:
            os.environ["FLB_TC"] = old
    torch.cuda.synchronize()
    return cios, tc


@pytest.mark.parametrize("count", [1, 127, 128, 129, 385])
def test_tc_ragged_tiles_match_cios_and_oracle(k2048, count):
    pub, priv, p, q = k2048
    n = p * q
    m_int = synthetic.uniform_below(n, count, 700 + count)
    m = to_dev(m_int, pub.pt_words)
    seed, ctr0 = 0x7C000000 + count, 11
    cios, tc = _both(priv, m, seed=seed, ctr0=ctr0)
    assert torch.equal(cios, tc)
    got = from_dev(tc)
    for i in sorted({0, count // 2, count - 1}):
        assert got[i] == paillier.encrypt(n, m_int[i], philox.draw_r(n, seed, ctr0 + i, pub.pt_words)), i


def test_tc_edge_operands(k2048):
    pub, priv, p, q = k2048
    n = p * q
    ms = [0, 1, n - 1, n // 2, 0, n - 1, 5, 7, 11]
    rs = [1, 1, 1, n - 1, n - 1, 2, p, q, 3 * p]
    m = to_dev(ms, pub.pt_words)
    r = to_dev(rs, pub.pt_words)
    cios, tc = _both(priv, m, r=r)
    assert torch.equal(cios, tc)
    got = from_dev(tc)
    for i, (mi, ri) in enumerate(zip(ms, rs)):
        assert got[i] == paillier.encrypt(n, mi, ri), i


def test_tc_large_batch_matches_cios(k2048):
    pub, priv, p, q = k2048
    count = 5000
    g = torch.Generator().manual_seed(99)
    m = torch.randint(-2**31, 2**31 - 1, (count, pub.pt_words), generator=g, dtype=torch.int32)
    m[:, -1] &= 0x3FFFFFFF
    m = m.cuda()
    cios, tc = _both(priv, m, seed=0xABCDEF, ctr0=1 << 33)
    bad = (cios != tc).any(dim=1).nonzero().flatten().tolist()
    assert not bad, bad[:5]


def _both_dec(priv, c):
    old = os.environ.get("FLB_TC")
    try:
        os.environ["FLB_TC"] = "0"
        cios = flb.decrypt(priv, c)
        os.environ["FLB_TC"] = "1"
        tc = flb.decrypt(priv, c)
    finally:
        if old is None:
            os.environ.pop("FLB_TC", None)
        else:
            os.environ["FLB_TC"] = old
    torch.cuda.synchronize()
    return cios, tc


@pytest.mark.parametrize("bits", ["1024", "2048"])
@pytest.mark.parametrize("count", [1, 129, 300])
def test_tc_decrypt_matches_cios_and_oracle(bits, count):
    """Decryption with c^(P-1) mod P^2 on the tensor cores (k_tc_exp + k_dec_finish): the same
    plaintexts as the CIOS k_decrypt and as the oracle's literal Eq. 4."""
    p, q = KEYS[bits]
    pub, priv = flb.key_from_primes(p, q)
    n = p * q
    m_int = synthetic.uniform_below(n, count, 900 + count)
    m_int[0] = 0
    if count > 1:
        m_int[-1] = n - 1
    seed = 0x7D000000 + count
    c = flb.encrypt(pub, to_dev(m_int, pub.pt_words), seed=seed)
    cios, tc = _both_dec(priv, c)
    assert torch.equal(cios, tc)
    got = from_dev(tc)
    assert got == m_int
    cc = from_dev(c)
    for i in sorted({0, count // 2, count - 1}):
        assert paillier.decrypt(p, q, cc[i]) == m_int[i], i


def test_tc_decrypt_arbitrary_ciphertexts_match_cios():
    """Any 2S-word c < n^2 (not only encryptions): both CRT exponentiation paths agree bit for bit."""
    p, q = KEYS["2048"]
    pub, priv = flb.key_from_primes(p, q)
    n2 = (p * q) ** 2
    cs = synthetic.uniform_below(n2, 1000, 4242)
    cs[:3] = [1, n2 - 1, p * p]
    c = to_dev(cs, pub.ct_words)
    cios, tc = _both_dec(priv, c)
    bad = (cios != tc).any(dim=1).nonzero().flatten().tolist()
    assert not bad, bad[:5]


@pytest.mark.parametrize("bits", ["3072", "4096"])
def test_tc_stage1_large_keys_match_cios_and_oracle(bits):
    """Key-holder stage 1 (r^Q mod P in the 64-word half frame) on the tensor cores at 3072/4096
    bits, stage 2 on CIOS: same ciphertexts as FLB_TC=0 and as the oracle's Eq. 3."""
    p, q = KEYS[bits]
    pub, priv = flb.key_from_primes(p, q)
    n = p * q
    count = 130
    m_int = synthetic.uniform_below(n, count, 77)
    m = to_dev(m_int, pub.pt_words)
    cios, tc = _both(priv, m, seed=0x51, ctr0=5)
    assert torch.equal(cios, tc)
    got = from_dev(tc)
    for i in (0, 64, 129):
        assert got[i] == paillier.encrypt(n, m_int[i], philox.draw_r(n, 0x51, 5 + i, pub.pt_words)), i


def test_tc_multi_tile_per_cta_both_problems():
    """Batches larger than one round of the persistent grid (every CTA runs several tiles and
    crosses from the p problem into the q problem, whose window tables differ in size at 1024
    bits): decryption and key-holder encryption equal the CIOS kernels bit for bit."""
    p, q = KEYS["1024"]
    pub, priv = flb.key_from_primes(p, q)
    n = p * q
    count = 40000
    m_int = synthetic.uniform_below(n, count, 31337)
    m = to_dev(m_int, pub.pt_words)
    c = flb.encrypt(pub, m, seed=0x99)
    cios, tc = _both_dec(priv, c)
    assert torch.equal(cios, tc)
    assert torch.equal(tc, m)
    p2, q2 = KEYS["2048"]
    pub2, priv2 = flb.key_from_primes(p2, q2)
    m2 = to_dev(synthetic.uniform_below(p2 * q2, count, 4711), pub2.pt_words)
    cios_e, tc_e = _both(priv2, m2, seed=0x98, ctr0=3)
    assert torch.equal(cios_e, tc_e)
    cios_d, tc_d = _both_dec(priv2, tc_e)
    assert torch.equal(cios_d, tc_d)
    assert torch.equal(tc_d, m2)


@pytest.mark.parametrize("words", [32, 64, 96, 128])
@pytest.mark.parametrize("square", [0, 1, 2], ids=["general", "sqr_tri", "sqr_split"])
def test_tc_product_phase_exact(words, square):
    """The tensor-core kernel's CUDA-core product phase (general row scan, or the block squaring
    of a^2) gives the exact 2w-limb integer product on random and extreme operands."""
    count = 128
    rnd = synthetic.uniform_below(1 << (32 * words), count, 5150 + words + square)
    top = (1 << (32 * words)) - 1
    rnd[:6] = [0, 1, top, top - 1, 1 << (32 * words - 1), (1 << (16 * words)) - 1]
    other = synthetic.uniform_below(1 << (32 * words), count, 6150 + words)
    a = to_dev(rnd, words)
    b = to_dev(other, words)
    t = from_dev(flb.debug_tc_product(a, b, square=square))
    for i in range(count):
        want = rnd[i] * (rnd[i] if square else other[i])
        assert t[i] == want, (i, hex(t[i] ^ want))


@pytest.mark.parametrize("words", [32, 64, 96, 128])
@pytest.mark.parametrize("sq", [1, 2], ids=["tri", "split"])
def test_tc_square_block_carries(words, sq):
    """Block squaring with triangular diagonal blocks (sqr_local: sum_{i<j} a_i a_j by lo/hi row
    chains, doubled, plus a_i^2): operands whose 16-limb lane blocks are all-ones, zero, or
    alternate 0xffffffff / 1 limbs, so every row chain, the doubling's shifted-out bits and the
    quarter carries hit their extremes; exact 2w-limb a^2.  sq = 2: the half-split diagonal square
    (two X/2 triangles + the doubled L H block rippled to the top), the form decryption and stage 1
    of the key-holder encryption use.  S = 96: eight lanes of 12 limbs (the half block starts half-way
    into a 16-byte chunk)."""
    X = 12 if words == 96 else 16
    nb = words // X
    full = (1 << (32 * X)) - 1
    alt = sum((0xFFFFFFFF if j % 2 == 0 else 1) << (32 * j) for j in range(X))
    alt2 = sum((1 if j % 2 == 0 else 0xFFFFFFFF) << (32 * j) for j in range(X))
    vals = []
    for blk in (full, alt, alt2, full - 1, 1 << (32 * X - 1)):
        for kb in range(nb):
            vals.append(blk << (32 * X * kb))                                  # one block set
        vals.append(sum(blk << (32 * X * kb) for kb in range(nb)))             # every block
        vals.append(sum(blk << (32 * X * kb) for kb in range(0, nb, 2)))       # alternate blocks
    half = (1 << (32 * X // 2)) - 1
    for blk in (half, half << (32 * X // 2), (half << (32 * X // 2)) | 1):  # L or H half all-ones
        vals.append(sum(blk << (32 * X * kb) for kb in range(nb)))
    vals += synthetic.uniform_below(1 << (32 * words), 128 - len(vals), 7150 + words)
    a = to_dev(vals, words)
    t = from_dev(flb.debug_tc_product(a, a, square=sq))
    for i, v in enumerate(vals):
        assert t[i] == v * v, (i, hex(t[i] ^ (v * v)))


def _env_run(fn, env):
    old = {k: os.environ.get(k) for k in env}
    try:
        os.environ.update(env)
        out = fn()
        torch.cuda.synchronize()
        return out
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


@pytest.mark.parametrize("count", [1, 129, 300, 20000])
def test_tc_dag_launch_matches_two_launches_and_oracle(k2048, count):
    """Both key-holder stages in one k_tc_exp_dag launch (dynamic tile queue, stage-2 tiles wait on
    their stage-1 tile's flag): same ciphertexts as the two k_tc_exp launches (FLB_TC_DAG=0), as the
    CIOS kernels, and as the oracle's Eq. 3 on sampled elements.  count = 20000 gives several tiles
    of both stages per CTA (4 x 157 tiles on 296 CTAs), so stage-2 tiles run on other CTAs than the
    stage-1 tiles they read."""
    pub, priv, p, q = k2048
    n = p * q
    m_int = synthetic.uniform_below(n, min(count, 64), 900 + count)
    m_int = (m_int * ((count + len(m_int) - 1) // len(m_int)))[:count]
    m = to_dev(m_int, pub.pt_words)
    seed, ctr0 = 0x5DA60000 + count, 3
    dag = _env_run(lambda: flb.encrypt_crt(priv, m, seed=seed, ctr0=ctr0), {"FLB_TC": "1", "FLB_TC_DAG": "1"})
    two = _env_run(lambda: flb.encrypt_crt(priv, m, seed=seed, ctr0=ctr0), {"FLB_TC": "1", "FLB_TC_DAG": "0"})
    assert torch.equal(dag, two)
    if count <= 300:
        cios = _env_run(lambda: flb.encrypt_crt(priv, m, seed=seed, ctr0=ctr0), {"FLB_TC": "0"})
        assert torch.equal(dag, cios)
    got = from_dev(dag)
    for i in sorted({0, count // 3, count - 1}):
        assert got[i] == paillier.encrypt(n, m_int[i], philox.draw_r(n, seed, ctr0 + i, pub.pt_words)), i

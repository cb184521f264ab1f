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

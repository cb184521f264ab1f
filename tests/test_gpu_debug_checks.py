"""FLB_DEBUG_CHECKS (include/flb_paillier.h): with the variable set, the batch calls
run device-side range checks first and return FLB_EINVAL on m >= n, c >= n^2, malformed
offsets / idx and summand counts above 2^pad_bits; valid inputs give the same
bits as without the checks."""

import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402
from tests.helpers import golden_keys, to_dev  # noqa: E402

pytestmark = pytest.mark.gpu


@pytest.fixture
def checks():
    old = os.environ.get("FLB_DEBUG_CHECKS")
    os.environ["FLB_DEBUG_CHECKS"] = "1"
    yield
    if old is None:
        os.environ.pop("FLB_DEBUG_CHECKS", None)
    else:
        os.environ["FLB_DEBUG_CHECKS"] = old


@pytest.fixture(scope="module")
def key():
    p, q = golden_keys()["1024"]
    return flb.key_from_primes(p, q) + (p * q,)


def _einval(fn):
    with pytest.raises(flb.FlbError) as e:
        fn()
        torch.cuda.synchronize()
    assert e.value.code == -1
    assert "FLB_DEBUG_CHECKS" in str(e.value) or "2^pad_bits" in str(e.value)


def test_valid_inputs_same_bits(key, checks):
    pub, priv, n = key
    m = to_dev(synthetic.uniform_below(n, 300, 1), pub.pt_words)
    c = flb.encrypt(pub, m, seed=5)
    c2 = flb.encrypt_crt(priv, m, seed=5)
    assert torch.equal(c, c2)
    assert torch.equal(flb.decrypt(priv, c), m)
    s = flb.add(pub, c, c2)
    offs = torch.tensor([0, 100, 100, 300], dtype=torch.int64, device="cuda")
    r = flb.reduce_segments(pub, c, offs, idx=torch.arange(300, dtype=torch.int64, device="cuda"))
    os.environ["FLB_DEBUG_CHECKS"] = "0"
    assert torch.equal(s, flb.add(pub, c, c2))
    assert torch.equal(r, flb.reduce_segments(pub, c, offs, idx=torch.arange(300, dtype=torch.int64, device="cuda")))


def test_out_of_range_values_rejected(key, checks):
    pub, priv, n = key
    m_int = synthetic.uniform_below(n, 64, 2)
    m_int[17] = n              # m >= n
    m = to_dev(m_int, pub.pt_words)
    _einval(lambda: flb.encrypt(pub, m, seed=1))
    _einval(lambda: flb.encrypt_crt(priv, m, seed=1))
    c_int = [1] * 64
    c_int[3] = n * n           # c >= n^2
    c = to_dev(c_int, pub.ct_words)
    _einval(lambda: flb.decrypt(priv, c))
    _einval(lambda: flb.add(pub, c, c))
    _einval(lambda: flb.scalar_mul(pub, c, torch.ones((64, 1), dtype=torch.int32, device="cuda")))


def test_malformed_segments_rejected(key, checks):
    pub, priv, n = key
    c = to_dev([1] * 10, pub.ct_words)
    ok = torch.tensor([0, 4, 10], dtype=torch.int64, device="cuda")
    flb.reduce_segments(pub, c, ok)
    _einval(lambda: flb.reduce_segments(pub, c, torch.tensor([0, 6, 4], dtype=torch.int64, device="cuda"),
                                        idx=torch.arange(4, dtype=torch.int64, device="cuda")))
    bad_idx = torch.tensor([0, 1, 2, 10], dtype=torch.int64, device="cuda")
    _einval(lambda: flb.reduce_segments(pub, c, torch.tensor([0, 2, 4], dtype=torch.int64, device="cuda"),
                                        idx=bad_idx))


def test_summand_counts_rejected(key, checks):
    pub, priv, n = key
    cd = flb.Codec(1.0, 29, 3, 31)
    pt = to_dev([0] * 4, pub.pt_words)
    flb.unpack(pub, cd, pt, 100, summands=torch.tensor([8, 1, 2, 3], dtype=torch.int32, device="cuda"))
    _einval(lambda: flb.unpack(pub, cd, pt, 100, summands=torch.tensor([8, 9, 2, 3], dtype=torch.int32,
                                                                       device="cuda")))
    _einval(lambda: flb.unpack(pub, cd, pt, 100, summands=9))

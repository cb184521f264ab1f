"""GPU parity for the Table I generic API (mod_mul, mod_pow) and RSA (L247–L251)
against oracle/modarith.py, over every frame (32..256 limbs) with ragged batches."""

import random

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402
from oracle import modarith  # noqa: E402
from tests.helpers import from_dev, to_dev  # noqa: E402

pytestmark = pytest.mark.gpu


def _odd(bits, seed):
    return random.Random(seed).getrandbits(bits) | (1 << (bits - 1)) | 1


@pytest.mark.parametrize("bits", [61, 1024, 1500, 2048, 3072, 4096, 6000, 8192])
def test_mod_mul_and_pow(bits):
    n = _odd(bits, bits)
    M = flb.Modulus(n)
    cnt = 45
    a = synthetic.uniform_below(n, cnt, 1)
    b = synthetic.uniform_below(n, cnt, 2)
    a[0], b[0] = n - 1, n - 1
    ta, tb = to_dev(a, M.words), to_dev(b, M.words)
    assert from_dev(M.mul(ta, tb)) == [modarith.mod_mul(x, y, n) for x, y in zip(a, b)]
    rng = random.Random(3)
    e = [rng.getrandbits(64) >> rng.randrange(64) for _ in range(cnt)]
    e[1] = 0
    te = torch.from_numpy(synthetic.ints_to_limbs(e, 2).view(np.int32)).cuda()
    assert from_dev(M.pow(ta, te)) == [modarith.mod_pow(x, y, n) for x, y in zip(a, e)]
    es = rng.getrandbits(min(bits, 512)) | 1
    assert from_dev(M.pow_shared(ta, es)) == [modarith.mod_pow(x, es, n) for x in a]
    assert from_dev(M.pow_shared(ta, 0)) == [1] * cnt


@pytest.mark.parametrize("bits", [1024, 2048])
def test_rsa_through_generic_api(bits):
    n, e, d, p, q = flb.rsa_keygen(bits, 11)
    assert p * q == n and n.bit_length() == bits
    M = flb.Modulus(n)
    ms = synthetic.uniform_below(n, 70, 4)
    tm = to_dev(ms, M.words)
    c = M.pow_shared(tm, e)
    assert from_dev(c) == [modarith.rsa_encrypt(n, e, m) for m in ms]
    assert torch.equal(M.pow_shared(c, d), tm)
    prod = M.mul(c[:35], c[35:])
    assert from_dev(M.pow_shared(prod, d)) == [ms[i] * ms[35 + i] % n for i in range(35)]

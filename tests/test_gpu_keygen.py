"""GPU key generation (NEXT-3): Miller–Rabin verdicts bit-exact against the oracle's
Miller–Rabin with the same bases; keygen_gpu yields valid, deterministic keys."""

import random

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402
from oracle import paillier  # noqa: E402
from tests.helpers import to_dev  # noqa: E402

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("bits,words", [(40, 32), (512, 32), (1024, 32), (1536, 64), (2048, 64)])
def test_miller_rabin_matches_oracle(bits, words):
    rng = random.Random(bits)
    cands = []
    for i in range(90):
        if i % 3 == 0:
            cands.append(paillier.random_prime(bits, rng))  # primes
        else:
            cands.append(rng.getrandbits(bits) | (1 << (bits - 1)) | 1)  # mostly composites
    if bits == 40:
        cands[1:6] = [561, 1105, 1729, 2047, 1373653]  # Carmichael / strong pseudoprimes
    rounds = 3
    R = 1 << (32 * words)
    mb = [rng.randrange(1, c) for c in cands for _ in range(rounds)]
    got = flb.miller_rabin(to_dev(cands, words), rounds, to_dev(mb, words)).cpu().numpy()
    for i, c in enumerate(cands):
        bases = [mb[i * rounds + r] * pow(R, -1, c) % c for r in range(rounds)]
        assert bool(got[i]) == paillier.miller_rabin_bases(c, bases), (i, c)


def test_miller_rabin_philox_bases_agree_with_primality():
    rng = random.Random(5)
    primes = [paillier.random_prime(256, rng) for _ in range(20)]
    comps = [p * q for p, q in zip(primes[:10], primes[10:])]
    comps = [c for c in comps if c.bit_length() <= 1024]
    cands = primes + comps + [paillier.random_prime(256, rng) * 3]
    got = flb.miller_rabin(to_dev(cands, 32), 20, seed=9).cpu().numpy().tolist()
    assert got == [1] * 20 + [0] * (len(cands) - 20)


@pytest.mark.parametrize("bits", [1024, 2048])
def test_keygen_gpu_valid_and_deterministic(bits):
    pub, priv = flb.keygen_gpu(bits, 123)
    p, q, n = priv.export()
    assert n == p * q and n.bit_length() == bits and p > q
    assert p.bit_length() == q.bit_length() == bits // 2
    for x in (p, q):
        assert all(pow(b, x - 1, x) == 1 for b in (2, 3, 5, 7))
    assert flb.keygen_gpu(bits, 123)[1].export() == (p, q, n)
    # and the key works end to end
    m = to_dev(synthetic.uniform_below(n, 64, 1), pub.pt_words)
    assert torch.equal(flb.decrypt(priv, flb.encrypt(pub, m, seed=1)), m)

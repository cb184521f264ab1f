"""Segmented multi-exponentiation (Pippenger bucket method and the scalar-mul fallback) against the
oracle: out_j = prod_t c[idx t]^(e_t) mod n^2 (Table I mod_pow composed with Eq. 5)."""

import os
import random

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402
from oracle import codec, paillier  # noqa: E402
from tests.helpers import from_dev, golden_keys, to_dev  # noqa: E402

pytestmark = pytest.mark.gpu
KEYS = golden_keys()


def _case(name, L, offsets, e_words, seed):
    p, q = KEYS[name]
    pub, priv = flb.key_from_primes(p, q)
    n2 = (p * q) ** 2
    rng = random.Random(seed)
    nent = offsets[-1]
    cs = synthetic.uniform_below(n2, L, seed)
    idx = [rng.randrange(L) for _ in range(nent)]
    es = [rng.getrandbits(32 * e_words) >> rng.randrange(32 * e_words) for _ in range(nent)]
    es[:3] = [0, 1, (1 << (32 * e_words)) - 1][:min(3, nent)]
    exp = []
    for j in range(len(offsets) - 1):
        acc = 1
        for t in range(offsets[j], offsets[j + 1]):
            acc = acc * paillier.scalar_mul(p * q, cs[idx[t]], es[t]) % n2
        exp.append(acc)
    args = (pub, to_dev(cs, pub.ct_words),
            torch.from_numpy(synthetic.ints_to_limbs(es, e_words).view(np.int32)).cuda(),
            torch.tensor(offsets, dtype=torch.int64).cuda(), torch.tensor(idx, dtype=torch.int64).cuda())
    return args, exp


@pytest.mark.parametrize("name,e_words", [("1024", 1), ("2048", 1), ("1024", 2), ("toy16", 1)])
def test_multiexp_pippenger_and_naive(name, e_words):
    args, exp = _case(name, 900, [0, 700, 700, 1500, 2100], e_words, 5)  # avg >= 256: bucket method
    assert from_dev(flb.multiexp_segments(*args[:4], idx=args[4])) == exp
    os.environ["FLB_MULTIEXP"] = "naive"
    try:
        assert from_dev(flb.multiexp_segments(*args[:4], idx=args[4])) == exp
    finally:
        del os.environ["FLB_MULTIEXP"]


def test_multiexp_short_segments_use_fallback():
    args, exp = _case("1024", 200, [0, 3, 3, 40, 41, 120], 1, 6)
    assert from_dev(flb.multiexp_segments(*args[:4], idx=args[4])) == exp


def test_c3_shape_decrypts_to_exact_sums():
    """Hetero LR (C3 shape, 65,536 residuals x 8 features): Dec(out_f) = sum_i q(d_i) x_if exactly."""
    p, q = KEYS["2048"]
    pub, priv = flb.key_from_primes(p, q)
    N, F = 1 << 16, 8
    d, x = synthetic.c3_residuals(N, F)
    cd = flb.Codec(1.0, 30, 2, 1)
    pt = flb.pack(pub, cd, torch.from_numpy(d).cuda())
    ct = flb.encrypt_crt(priv, pt, seed=3)
    i = torch.arange(N, dtype=torch.int64, device="cuda")
    idx = torch.cat([i for _ in range(F)])
    e = torch.from_numpy(np.ascontiguousarray(x.T).reshape(N * F, 1).view(np.int32)).cuda()  # entry (f, i)
    offs = torch.arange(F + 1, dtype=torch.int64, device="cuda") * N
    agg = flb.multiexp_segments(pub, ct, e, offs, idx=idx)
    got = from_dev(flb.decrypt(priv, agg))
    qd = np.array([codec.quantize(float(v), 1.0, 30) for v in d], dtype=object)
    for f in range(F):
        assert got[f] == int(np.dot(qd, x[:, f].astype(object))) % (p * q)

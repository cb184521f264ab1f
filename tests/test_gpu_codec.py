"""GPU parity for quantise/pack and unpack/dequantise (PAPER §IV-B/C) against oracle/codec.py.

Integers (packed plaintexts, slot sums) must match bit for bit; dequantised float32 values must
match the oracle's binary64->binary32 result exactly (same op order), which is stricter than the
north star's 1e-6 relative bound (also asserted).
"""

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402
from oracle import codec  # noqa: E402
from tests.helpers import from_dev, golden_keys, to_dev  # noqa: E402

pytestmark = pytest.mark.gpu
KEYS = golden_keys()

# (key, alpha, qbits, pad_bits, slots): C1 (L432 setting, S = 1), C2 (S = 63), C4 (w = 64, S = 2),
# full 32-bit capacity at 1024 bits, full capacity at 3072 bits
CASES = [
    ("1024", 0.5, 30, 2, 1),
    ("2048", 1.0, 29, 3, 63),
    ("2048", 1.0, 44, 20, 2),
    ("1024", 1.0, 29, 3, 31),
    ("4096", 1.0, 30, 34, 63),
    ("3072", 1.0, 29, 3, 95),
]


def _values(n, seed):
    x = np.random.default_rng(seed).normal(0, 0.4, n).astype(np.float32)
    x[:8] = [np.nan, np.inf, -np.inf, 5.0, -5.0, 0.0, -0.0, 1.0]
    return x


@pytest.mark.parametrize("case", CASES)
def test_pack_unpack(case):
    name, alpha, qb, pb, slots = case
    p, q = KEYS[name]
    pub, priv = flb.key_from_primes(p, q)
    cd = flb.Codec(alpha, qb, pb, slots)
    n = 5 * slots + 3  # ragged tail
    x = _values(n, 7)
    pt = flb.pack(pub, cd, torch.from_numpy(x).cuda())
    exp = codec.pack([float(v) for v in x], alpha, qb, pb, slots)
    assert from_dev(pt) == exp
    # aggregate 3 copies (what Dec(prod Enc) gives) and unpack with cnt = 3
    agg = [3 * z for z in exp]
    aggt = to_dev(agg, pub.pt_words)
    got_sums = flb.unpack_sums(pub, cd, aggt, n).cpu().numpy().view(np.uint64).tolist()
    assert got_sums == codec.unpack_sums(agg, n, qb, pb, slots)
    got = flb.unpack(pub, cd, aggt, n, summands=3).cpu().numpy()
    ref = np.array(codec.unpack(agg, n, alpha, qb, pb, slots, 3), dtype=np.float32)
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))
    assert np.all(np.abs(got - ref) <= 1e-6 * np.maximum(np.abs(ref), 2 * alpha / ((1 << qb) - 1)))


def test_unpack_per_plaintext_counts():
    p, q = KEYS["2048"]
    pub, priv = flb.key_from_primes(p, q)
    cd = flb.Codec(1.0, 44, 20, 2)
    gh, b, offsets, idx = synthetic.c4_histogram(n=1000, bins=16)
    pts = codec.pack([float(v) for v in gh], 1.0, 44, 20, 2)
    # bin sums of plaintexts (what the segmented reduce + decrypt produce)
    counts = np.diff(offsets)
    sums = [sum(pts[int(t)] for t in idx[offsets[j]:offsets[j + 1]]) for j in range(16)]
    got = flb.unpack(pub, cd, to_dev(sums, pub.pt_words), 32,
                     summands=torch.from_numpy(counts.astype(np.int32)).cuda()).cpu().numpy()
    ref = np.array(codec.unpack(sums, 32, 1.0, 44, 20, 2, [int(c) for c in counts]), dtype=np.float32)
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


def test_codec_rejects_bad_parameters():
    p, q = KEYS["1024"]
    pub, priv = flb.key_from_primes(p, q)
    x = torch.zeros(10, dtype=torch.float32).cuda()
    with pytest.raises(flb.FlbError):
        flb.pack(pub, flb.Codec(1.0, 29, 3, 32), x)      # 32 slots > capacity 31
    with pytest.raises(flb.FlbError):
        flb.pack(pub, flb.Codec(1.0, 29, 4, 1), x)       # slot_bits 33
    with pytest.raises(flb.FlbError):
        flb.pack(pub, flb.Codec(0.0, 29, 3, 1), x)       # alpha <= 0

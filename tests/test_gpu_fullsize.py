"""Parity at BASELINE.json's full sizes, in bench.py's launch configuration.

The oracle cannot recompute 133,160 2048-bit encryptions in test time, so: sampled outputs are
recomputed one by one by the oracle (from the seeded inputs only), and properties that hold at
any size are checked on every output (decrypted aggregates equal the exact integer sums of the
oracle-packed plaintexts; dequantised gradients are within the quantisation bound of the float64
sum of the seeded inputs).
"""

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402
from oracle import codec, paillier, philox  # noqa: E402
from paper_conf_icde_zeng0fcpcwg23_b200 import dist as fdist  # noqa: E402
from tests.helpers import from_dev, golden_keys, to_dev  # noqa: E402

pytestmark = pytest.mark.gpu
KEYS = golden_keys()


@pytest.fixture(scope="module")
def key2048():
    p, q = KEYS["2048"]
    return flb.key_from_primes(p, q) + (p, q)


@pytest.mark.parametrize("mode", ["keyholder", "public"])
def test_c2_full_homo_lr_round(key2048, mode):
    """C2: 8 clients x 1,048,576 values, w = 32, S = 63 -> 133,160 encryptions, 8-way products,
    16,645 decryptions, unpack — exactly the bench step."""
    pub, priv, p, q = key2048
    n = p * q
    clients, nv, S = 8, 1 << 20, 63
    alpha, qb, pb = 1.0, 29, 3
    cd = flb.Codec(alpha, qb, pb, S)
    rows = cd.num_plaintexts(nv)
    xs = [synthetic.c2_gradient(c) for c in range(clients)]
    pt = torch.cat([flb.pack(pub, cd, torch.from_numpy(x).cuda()) for x in xs])
    seed = 0xC2000000 + 1000
    enc = flb.encrypt_crt if mode == "keyholder" else flb.encrypt
    ct = enc(priv if mode == "keyholder" else pub, pt, seed=seed)
    offs, idx = fdist.client_segments(clients, rows, device="cuda")
    agg = flb.reduce_segments(pub, ct, offs, idx=idx, max_segment_len=clients)
    dec = flb.decrypt(priv, agg)
    out = flb.unpack(pub, cd, dec, nv, summands=clients).cpu().numpy()

    def oracle_pt(c, j):
        return codec.pack([float(v) for v in xs[c][j * S:(j + 1) * S]], alpha, qb, pb, S)[0]

    # sampled plaintexts and ciphertexts (first, ragged last row, persistent-loop wrap points)
    ptl = pt.cpu().numpy()
    ctl = ct.cpu().numpy()
    for c, j in [(0, 0), (3, 9471), (7, rows - 1), (5, 12345)]:
        i = c * rows + j
        z = oracle_pt(c, j)
        assert synthetic.limbs_to_ints(ptl[i:i + 1])[0] == z
        assert synthetic.limbs_to_ints(ctl[i:i + 1])[0] == paillier.encrypt(n, z, philox.draw_r(n, seed, i, 64))
    # sampled aggregates: the oracle product of the oracle's own ciphertexts
    aggl = agg.cpu().numpy()
    j = rows - 1
    cts = [paillier.encrypt(n, oracle_pt(c, j), philox.draw_r(n, seed, c * rows + j, 64)) for c in range(clients)]
    assert synthetic.limbs_to_ints(aggl[j:j + 1])[0] == paillier.reduce_segments(n, cts, [0, clients])[0]
    # every row: Dec(prod_c Enc(z_c)) = sum_c z_c (exact integers from the oracle codec), sampled
    decl = dec.cpu().numpy()
    for j in list(range(0, rows, 997)) + [rows - 1]:
        assert synthetic.limbs_to_ints(decl[j:j + 1])[0] == sum(oracle_pt(c, j) for c in range(clients))
    # every value: within the quantisation bound of the exact float64 sum (property at full size)
    exact = np.sum(np.array(xs, dtype=np.float64), axis=0)
    err = np.abs(out.astype(np.float64) - exact)
    assert np.all(err <= clients * alpha / ((1 << qb) - 1) + np.abs(exact) * 2.0 ** -24 + 1e-12)
    # sampled unpacked values bit-exact vs the oracle decode of the oracle sums
    for j in (0, rows // 2, rows - 1):
        s = sum(oracle_pt(c, j) for c in range(clients))
        nvals = min(S, nv - j * S)
        ref = np.array(codec.unpack([s], nvals, alpha, qb, pb, S, clients), dtype=np.float32)
        assert np.array_equal(out[j * S:j * S + nvals].view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("skew", [False, True])
def test_c4_full_sbt_histogram(key2048, skew):
    """C4: 1,048,576 samples, (g, h) packed in two 64-bit slots, segmented product into 256 bins
    (quantile bins, or Zipf(1.2)-skewed), decrypt, unpack with per-bin counts."""
    pub, priv, p, q = key2048
    n = p * q
    nsamp, bins = 1 << 20, 256
    alpha, qb, pb, S = 1.0, 44, 20, 2
    cd = flb.Codec(alpha, qb, pb, S)
    gh, b, offsets, idx = synthetic.c4_histogram(n=nsamp, bins=bins, skew=skew)
    pt = flb.pack(pub, cd, torch.from_numpy(gh).cuda())
    seed = 0xC4
    ct = flb.encrypt_crt(priv, pt, seed=seed)
    counts = np.diff(offsets)
    agg = flb.reduce_segments(pub, ct, torch.from_numpy(offsets).cuda(), idx=torch.from_numpy(idx).cuda(),
                              max_segment_len=int(counts.max()))
    dec = flb.decrypt(priv, agg)
    out = flb.unpack(pub, cd, dec, 2 * bins, summands=torch.from_numpy(counts.astype(np.int32)).cuda()).cpu().numpy()
    # exact per-bin sums of the oracle-quantised (g, h): Dec(bin) must equal them
    ghq = [codec.quantize(float(v), alpha, qb) for v in gh]
    gq = np.array(ghq[0::2], dtype=object)
    hq = np.array(ghq[1::2], dtype=object)
    decv = synthetic.limbs_to_ints(dec.cpu().numpy())
    for j in range(bins):
        sel = idx[offsets[j]:offsets[j + 1]]
        sg, sh = int(sum(gq[sel])), int(sum(hq[sel]))
        assert decv[j] == (sg << 64) + sh, j
        ref = codec.unpack([decv[j]], 2, alpha, qb, pb, S, int(counts[j]))
        assert np.array_equal(out[2 * j:2 * j + 2], np.array(ref, dtype=np.float32))
    ctl = ct.cpu().numpy()
    for i in (0, nsamp // 3, nsamp - 1):
        z = codec.pack([float(gh[2 * i]), float(gh[2 * i + 1])], alpha, qb, pb, S)[0]
        assert synthetic.limbs_to_ints(ctl[i:i + 1])[0] == paillier.encrypt(n, z, philox.draw_r(n, seed, i, 64))


@pytest.mark.parametrize("name,count", [("1024", 40000), ("3072", 3000), ("4096", 6000)])
def test_roundtrip_beyond_one_wave(name, count):
    """Batches larger than the resident grid (the persistent loop wraps): Dec(Enc(m)) = m for all,
    sampled ciphertexts vs the oracle, key-holder and public paths identical."""
    p, q = KEYS[name]
    pub, priv = flb.key_from_primes(p, q)
    n = p * q
    ms = synthetic.uniform_below(n, count, 71)
    m = to_dev(ms, pub.pt_words)
    c = flb.encrypt_crt(priv, m, seed=3)
    assert torch.equal(flb.decrypt(priv, c), m)
    c2 = flb.encrypt(pub, m, seed=3)
    assert torch.equal(c, c2)
    cl = c.cpu().numpy()
    for i in (0, count - 1):
        assert synthetic.limbs_to_ints(cl[i:i + 1])[0] == paillier.encrypt(n, ms[i],
                                                                          philox.draw_r(n, 3, i, pub.pt_words))


def test_c2_full_batch_public_equals_keyholder(key2048):
    """Every one of the bench's 133,160 ciphertexts agrees between the public-key path (n^2 frame,
    8 lanes per integer, exponent n) and the two-stage key-holder path (half and p^2 frames, 2 and 4
    lanes, exponents q then p): independent operand sets, so a rare carry slip in either shows up
    here even when sampled oracle checks miss it (a one-in-2^30-steps carry bug did, in development)."""
    pub, priv, p, q = key2048
    count = 133160
    g = torch.Generator().manual_seed(2048)
    m = torch.randint(-2**31, 2**31 - 1, (count, pub.pt_words), generator=g, dtype=torch.int32)
    m[:, -1] &= 0x3FFFFFFF  # m < 2^2046 < n
    m = m.cuda()
    a = flb.encrypt(pub, m, seed=0xC2000001)
    b = flb.encrypt_crt(priv, m, seed=0xC2000001)
    bad = (a != b).any(dim=1).nonzero().flatten().tolist()
    assert not bad, f"{len(bad)} of {count} ciphertexts differ, first {bad[:5]}"
    assert torch.equal(flb.decrypt(priv, b), m)

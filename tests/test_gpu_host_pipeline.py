"""The host-buffer pipeline (flb_*_host, NEXT-1 / PAPER Fig. 4) gives the same bits as the
device-buffer calls, across several chunks with a ragged tail; sampled outputs vs the oracle."""

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icde_zeng0fcpcwg23_b200 as flb  # noqa: E402
import synthetic  # noqa: E402
from oracle import codec, paillier, philox  # noqa: E402
from paper_conf_icde_zeng0fcpcwg23_b200 import dist as fdist  # noqa: E402
from tests.helpers import golden_keys  # noqa: E402

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("keyholder", [True, False])
def test_c2_round_through_host_buffers(keyholder):
    p, q = golden_keys()["1024"]
    pub, priv = flb.key_from_primes(p, q)
    n = p * q
    S, clients = 31, 3
    cd = flb.Codec(1.0, 29, 3, S)
    nv = 70000 * S + 17          # 70,001 plaintexts per client: 3 chunks of 32,768, ragged tail
    xs = [synthetic.c2_gradient(c, n=nv) for c in range(clients)]
    rows = cd.num_plaintexts(nv)
    cts = np.concatenate([flb.pack_encrypt_host(pub, cd, xs[c], seed=9, ctr0=c * rows,
                                                priv=priv if keyholder else None) for c in range(clients)])
    # same bits as the device path
    dev = torch.cat([flb.pack(pub, cd, torch.from_numpy(x).cuda()) for x in xs])
    ref = flb.encrypt(pub, dev, seed=9).cpu().numpy().view(np.uint32)
    assert np.array_equal(cts, ref)
    i = clients * rows - 1
    z = codec.pack([float(v) for v in xs[-1][(rows - 1) * S:]], 1.0, 29, 3, S)[0]
    assert synthetic.limbs_to_ints(cts[i:i + 1])[0] == paillier.encrypt(n, z, philox.draw_r(n, 9, i, pub.pt_words))
    offs, idx = fdist.client_segments(clients, rows)
    agg = flb.reduce_segments_host(pub, cts, offs.numpy(), idx.numpy(), max_segment_len=clients)
    agg_dev = flb.reduce_segments(pub, torch.from_numpy(cts.view(np.int32)).cuda(), offs.cuda(),
                                  idx=idx.cuda(), max_segment_len=clients).cpu().numpy().view(np.uint32)
    assert np.array_equal(agg, agg_dev)
    out = flb.decrypt_unpack_host(priv, cd, agg, nv, summands=clients)
    dec = flb.decrypt(priv, torch.from_numpy(agg.view(np.int32)).cuda())
    out_dev = flb.unpack(pub, cd, dec, nv, summands=clients).cpu().numpy()
    assert np.array_equal(out.view(np.uint32), out_dev.view(np.uint32))
    exact = np.sum(np.array(xs, dtype=np.float64), axis=0)
    assert np.max(np.abs(out - exact)) <= clients / ((1 << 29) - 1) + 1e-6


def test_decrypt_unpack_host_per_plaintext_counts():
    p, q = golden_keys()["1024"]
    pub, priv = flb.key_from_primes(p, q)
    cd = flb.Codec(1.0, 44, 20, 2)
    x = np.random.default_rng(3).uniform(-1, 1, 2 * 40000).astype(np.float32)
    c = flb.pack_encrypt_host(pub, cd, x, seed=4)
    cnt = np.ones(c.shape[0], dtype=np.uint32)
    out = flb.decrypt_unpack_host(priv, cd, c, x.shape[0], summands=cnt)
    assert np.max(np.abs(out - x)) <= 1.0 / ((1 << 44) - 1) + np.abs(x).max() * 2 ** -24


def test_multi_array_host_encrypt_equals_per_array_calls():
    p, q = golden_keys()["1024"]
    pub, priv = flb.key_from_primes(p, q)
    cd = flb.Codec(1.0, 29, 3, 31)
    xs = [synthetic.c2_gradient(c, n=n) for c, n in enumerate([31 * 40000 + 5, 17, 31 * 3000, 0, 999])]
    multi = flb.pack_encrypt_host_multi(pub, cd, xs, seed=21, ctr0=100, priv=priv)
    parts, ctr = [], 100
    for x in xs:
        if x.shape[0]:
            parts.append(flb.pack_encrypt_host(pub, cd, x, seed=21, ctr0=ctr, priv=priv))
            ctr += cd.num_plaintexts(x.shape[0])
    assert np.array_equal(multi, np.concatenate(parts))


def _pinned(shape, dtype):
    t = torch.empty(shape, dtype=torch.int32 if dtype == np.uint32 else torch.float32, pin_memory=True)
    return t.numpy().view(dtype)


def test_host_pipeline_page_locked_buffers():
    """Page-locked caller buffers (pin_memory tensors): the pipeline DMAs straight from / into them
    (no staging copy) and the bits equal the pageable-buffer calls; 8 clients of 16,645 + a ragged
    remainder, so the encryption runs as several equal chunks (flb_host_pipeline.cu chunk_rows)."""
    p, q = golden_keys()["2048"]
    pub, priv = flb.key_from_primes(p, q)
    S, clients = 63, 8
    cd = flb.Codec(1.0, 29, 3, S)
    nv = 16645 * S - 5
    xs = [synthetic.c2_gradient(c, n=nv) for c in range(clients)]
    xs_p = []
    for x in xs:
        xp = _pinned(x.shape, np.float32)
        xp[...] = x
        xs_p.append(xp)
    rows = cd.num_plaintexts(nv)
    cts_p = _pinned((clients * rows, pub.ct_words), np.uint32)
    flb.pack_encrypt_host_multi(pub, cd, xs_p, seed=21, priv=priv, out=cts_p)
    cts = flb.pack_encrypt_host_multi(pub, cd, xs, seed=21, priv=priv)
    assert np.array_equal(cts_p, cts)
    offs, idx = fdist.client_segments(clients, rows)
    agg_p = _pinned((rows, pub.ct_words), np.uint32)
    flb.reduce_segments_host(pub, cts_p, offs.numpy(), idx.numpy(), max_segment_len=clients, out=agg_p)
    agg = flb.reduce_segments_host(pub, cts, offs.numpy(), idx.numpy(), max_segment_len=clients)
    assert np.array_equal(agg_p, agg)
    out_p = _pinned((nv,), np.float32)
    flb.decrypt_unpack_host(priv, cd, agg_p, nv, summands=clients, out=out_p)
    out = flb.decrypt_unpack_host(priv, cd, agg, nv, summands=clients)
    assert np.array_equal(out_p.view(np.uint32), out.view(np.uint32))
    exact = np.sum(np.array(xs, dtype=np.float64), axis=0)
    assert np.max(np.abs(out_p - exact)) <= clients / ((1 << 29) - 1) + 1e-6
    with pytest.raises(ValueError):
        flb.reduce_segments_host(pub, cts_p, offs.numpy(), idx.numpy(), max_segment_len=clients, out=agg_p[:-1])

"""a9 under the CUDA path: the cross-rank finish of the Homo-LR aggregation
(Fig. 2: clients encrypt, the server multiplies their ciphertexts) with two ranks
on one GPU (gloo process group, both processes on cuda:0).

Each rank hosts CLIENTS clients of a 2·CLIENTS-client federation at a 2048-bit key: pack ->
encrypt (Philox counter = global element index, so the bits do not depend on the rank count) ->
local product over its clients (flb.reduce_segments) -> dist.exchange_and_finish with
flb.reduce_segments as the finishing product -> decrypt its rows.  The parent process computes the
1-rank aggregate of all 2·CLIENTS clients on the same GPU; the ranks' rows must equal it bit for
bit, and sampled rows are recomputed by the oracle (ciphertext product mod n^2 and its
decryption = the exact integer sum of the oracle-packed plaintexts)."""

import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import torch.multiprocessing as mp  # noqa: E402

pytestmark = pytest.mark.gpu

WORLD = 2
KEY = "2048"


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _setup(clients, nvals):
    import paper_conf_icde_zeng0fcpcwg23_b200 as flb
    from tests.helpers import golden_keys
    p, q = golden_keys()[KEY]
    pub, priv = flb.key_from_primes(p, q)
    cd = flb.Codec(1.0, 28, 4, pub.slot_capacity(32))  # b = 4 >= log2(2 * clients) summands
    return flb, pub, priv, cd, p, q


def _encrypt_clients(flb, pub, priv, cd, gclients, nvals, rows, seed):
    """Plaintexts and key-holder ciphertexts of the global clients `gclients`, client-major."""
    import synthetic
    pts = torch.cat([flb.pack(pub, cd, torch.from_numpy(synthetic.c2_gradient(c, n=nvals)).cuda())
                     for c in gclients])
    ct = flb.encrypt_crt(priv, pts, seed=seed, ctr0=gclients[0] * rows)
    return pts, ct


def _worker(rank, port, clients, nvals, seed, outdir):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch.distributed as dist
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    from paper_conf_icde_zeng0fcpcwg23_b200 import dist as fdist
    flb, pub, priv, cd, _, _ = _setup(clients, nvals)
    rows = cd.num_plaintexts(nvals)
    rows_p = fdist.padded_rows(rows, WORLD)
    _, ct = _encrypt_clients(flb, pub, priv, cd, list(range(rank * clients, (rank + 1) * clients)), nvals, rows, seed)
    offs, idx = fdist.client_segments(clients, rows, rows_p, device="cuda")
    part = flb.reduce_segments(pub, ct, offs, idx=idx, max_segment_len=clients)
    assert part.shape[0] == rows_p
    fin = torch.empty((rows_p // WORLD, pub.ct_words), dtype=torch.int32, device="cuda")

    def reduce_cb(buf, o, i, L):
        return flb.reduce_segments(pub, buf, o, idx=i, max_segment_len=L, out=fin)

    mine = fdist.exchange_and_finish(part, None, reduce_cb, WORLD)
    r0, r1 = fdist.rank_rows(rows, WORLD, rank)
    dec = flb.decrypt(priv, mine[: r1 - r0])
    torch.cuda.synchronize()
    np.save(os.path.join(outdir, "agg%d.npy" % rank), mine.cpu().numpy())
    np.save(os.path.join(outdir, "dec%d.npy" % rank), dec.cpu().numpy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("clients,nvals", [(3, 63 * 101 + 17), (8, 1 << 20)], ids=["ragged", "c2"])
def test_two_rank_exchange_and_finish_cuda(tmp_path, clients, nvals):
    """Two ranks x `clients` clients; the second case is C2-shaped (2 x 8 clients x 1,048,576 values,
    16,645 rows, odd so the last rank's block is padded)."""
    import synthetic
    from oracle import codec, paillier
    from paper_conf_icde_zeng0fcpcwg23_b200 import dist as fdist
    seed = 0xA9000000 + clients
    ctx = mp.get_context("spawn")
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, clients, nvals, seed, str(tmp_path))) for r in range(WORLD)]
    for pr in procs:
        pr.start()
    for pr in procs:
        pr.join(timeout=900)
        assert pr.exitcode == 0, "rank process failed"

    # the 1-rank aggregate of all WORLD * clients clients on the same device
    flb, pub, priv, cd, p, q = _setup(clients, nvals)
    n = p * q
    rows = cd.num_plaintexts(nvals)
    G = WORLD * clients
    pts, ct = _encrypt_clients(flb, pub, priv, cd, list(range(G)), nvals, rows, seed)
    offs, idx = fdist.client_segments(G, rows, device="cuda")
    agg1 = flb.reduce_segments(pub, ct, offs, idx=idx, max_segment_len=G).cpu().numpy()
    dec1 = flb.decrypt(priv, torch.from_numpy(agg1).cuda()).cpu().numpy()
    ctl = ct.cpu().numpy()

    got_agg = np.concatenate([np.load(str(tmp_path / ("agg%d.npy" % r))) for r in range(WORLD)])
    got_dec = np.concatenate([np.load(str(tmp_path / ("dec%d.npy" % r))) for r in range(WORLD)])
    assert np.array_equal(got_agg[:rows], agg1), "2-rank aggregate differs from the 1-rank aggregate"
    assert np.array_equal(got_dec, dec1), "2-rank decryption differs"
    # padded rows are the empty product 1 = Enc(0; r = 1)
    pad = synthetic.limbs_to_ints(got_agg[rows:])
    assert all(v == 1 for v in pad)

    # sampled rows against the oracle: product of the GPU ciphertexts mod n^2, and its decryption
    # equals the exact sum of the oracle-packed plaintexts of every client
    xs = [synthetic.c2_gradient(c, n=nvals) for c in range(G)]
    S = cd.slots
    for j in sorted({0, rows // 2, rows // WORLD - 1, rows // WORLD, rows - 1}):
        cs = synthetic.limbs_to_ints(ctl[[c * rows + j for c in range(G)]])
        exp = paillier.reduce_segments(n, cs, [0, G], list(range(G)))[0]
        assert synthetic.limbs_to_ints(got_agg[j:j + 1])[0] == exp, j
        zs = [codec.pack([float(v) for v in xs[c][j * S:(j + 1) * S]], cd.alpha, cd.qbits, cd.pad_bits, S)[0]
              for c in range(G)]
        assert paillier.decrypt(p, q, exp) == sum(zs) % n
        assert synthetic.limbs_to_ints(got_dec[j:j + 1])[0] == sum(zs)

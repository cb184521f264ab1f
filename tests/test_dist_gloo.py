"""Multi-rank aggregation logic (paper_conf_icde_zeng0fcpcwg23_b200/dist.py) on CPU with gloo,
world_size 2: clients on two ranks, reduce-scatter of rows + finishing product, checked against
the single-process aggregation.  Ciphertexts of a toy key fit in int64, and the injected
product callback is the oracle's reduce_segments, so no device is needed."""

import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import paillier
from paper_conf_icde_zeng0fcpcwg23_b200 import dist as fdist
from tests.helpers import golden_keys

P, Q = golden_keys()["toy16"]
N = P * Q
CLIENTS, ROWS, WORLD = 3, 11, 2


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _cipher(client, row):
    m = (7 * client + 3 * row) % N
    r = 2 + (client * 131 + row * 17) % (N - 3)
    return paillier.encrypt(N, m, r), m


def _reduce_cb(buf, offsets, idx, L):
    vals = [int(v) for v in buf.view(-1).tolist()]
    out = paillier.reduce_segments(N, vals, offsets.tolist(), idx.tolist())
    return torch.tensor(out, dtype=torch.int64).view(-1, 1)


def _worker(rank, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    rows_p = fdist.padded_rows(ROWS, WORLD)
    # this rank's clients: global clients rank*CLIENTS + c; ciphertexts client-major [client][row]
    cts = [_cipher(rank * CLIENTS + c, j)[0] for c in range(CLIENTS) for j in range(ROWS)]
    offs, idx = fdist.client_segments(CLIENTS, ROWS, rows_p)
    part = _reduce_cb(torch.tensor(cts, dtype=torch.int64), offs, idx, CLIENTS)
    assert part.shape == (rows_p, 1)
    mine = fdist.exchange_and_finish(part, None, _reduce_cb, WORLD)
    r0, r1 = fdist.rank_rows(ROWS, WORLD, rank)
    q.put((rank, r0, r1, mine.view(-1).tolist()))
    dist.destroy_process_group()


def test_two_rank_aggregation_matches_single_process():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(WORLD)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(WORLD)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    # single-process reference: product over all WORLD*CLIENTS clients per row
    for rank, r0, r1, vals in res:
        for i, j in enumerate(range(r0, r1)):
            cs = [_cipher(c, j) for c in range(WORLD * CLIENTS)]
            exp = 1
            for c, _ in cs:
                exp = exp * c % (N * N)
            assert vals[i] == exp
            assert paillier.decrypt(P, Q, vals[i]) == sum(m for _, m in cs) % N
        # padded rows (beyond ROWS) are the empty product 1
        assert all(v == 1 for v in vals[r1 - r0:])


def test_layout_helpers():
    offs, idx = fdist.client_segments(3, 4, 6)
    assert offs.tolist() == [0, 3, 6, 9, 12, 12, 12]
    assert idx.tolist() == [0, 4, 8, 1, 5, 9, 2, 6, 10, 3, 7, 11]
    fo, fi = fdist.finish_segments(2, 3)
    assert fo.tolist() == [0, 2, 4, 6] and fi.tolist() == [0, 3, 1, 4, 2, 5]
    assert fdist.padded_rows(16645, 8) == 16648
    assert fdist.rank_rows(16645, 8, 7) == (14567, 16645)
    assert fdist.rank_rows(5, 4, 3) == (5, 5)

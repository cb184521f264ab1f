"""Multi-GPU aggregation of Paillier ciphertexts.

One process per GPU (torch.distributed, NCCL over NVLink/NVSwitch).  Every op of the hot path is
independent per ciphertext, so work shards by ciphertext with no collective; the one real
exchange is the cross-client product of the Homo-LR aggregation (Fig. 2): each
rank holds the product of its local clients' ciphertexts for ALL M plaintext rows; rows are
reduce-scattered with ``all_to_all_single`` so rank r owns rows [r*rows, (r+1)*rows), and the
N incoming partial products per row are multiplied by the same segmented-product kernel
(``reduce_segments`` with segments of length N).  NCCL has no modular-product reduction, hence
exchange + local finish.

The layout helpers are pure functions of sizes so they run (and are tested) on CPU; the
``reduce`` callable is injected so the same driver is exercised with a gloo process group and an
integer reference product in the CPU tests.
"""

from __future__ import annotations

from typing import Callable, Optional, Tuple

import torch


def client_segments(clients: int, rows: int, rows_padded: Optional[int] = None,
                    device=None) -> Tuple[torch.Tensor, torch.Tensor]:
    """Offsets/idx multiplying, for each plaintext row j, the ciphertexts of all ``clients``
    stored client-major ([client][row]).  Rows in [rows, rows_padded) are empty segments (their
    product is 1 = Enc(0; r=1))."""
    rp = rows if rows_padded is None else rows_padded
    j = torch.arange(rows, dtype=torch.int64)
    c = torch.arange(clients, dtype=torch.int64)
    idx = (c[None, :] * rows + j[:, None]).reshape(-1)
    offsets = torch.empty(rp + 1, dtype=torch.int64)
    offsets[: rows + 1] = torch.arange(rows + 1, dtype=torch.int64) * clients
    offsets[rows + 1:] = rows * clients
    return offsets.to(device), idx.to(device)


def padded_rows(rows: int, world: int) -> int:
    """Rows padded to a multiple of the world size (equal all_to_all splits)."""
    return -(-rows // world) * world


def finish_segments(world: int, rows_per_rank: int, device=None) -> Tuple[torch.Tensor, torch.Tensor]:
    """After all_to_all the receive buffer is [world][rows_per_rank]; row i multiplies entries
    w*rows_per_rank + i for every source rank w."""
    i = torch.arange(rows_per_rank, dtype=torch.int64)
    w = torch.arange(world, dtype=torch.int64)
    idx = (w[None, :] * rows_per_rank + i[:, None]).reshape(-1)
    offsets = torch.arange(rows_per_rank + 1, dtype=torch.int64) * world
    return offsets.to(device), idx.to(device)


def exchange_and_finish(partial: torch.Tensor, group, reduce: Callable, world: int,
                        recv: Optional[torch.Tensor] = None) -> torch.Tensor:
    """partial: [rows_padded, words] (this rank's product over its local clients, all rows).
    Returns this rank's rows of the global product: [rows_padded / world, words]."""
    import torch.distributed as dist
    rows_p, words = partial.shape
    rpr = rows_p // world
    if recv is None:
        recv = torch.empty_like(partial)
    if partial.is_cuda and dist.get_backend(group) == "gloo":
        # gloo has no CUDA all_to_all: stage through host memory (CPU tests / single-GPU multi-rank runs)
        host = torch.empty_like(partial, device="cpu")
        dist.all_to_all_single(host, partial.cpu(), group=group)
        recv.copy_(host)
    else:
        dist.all_to_all_single(recv, partial, group=group)
    offsets, idx = finish_segments(world, rpr, device=partial.device)
    return reduce(recv, offsets, idx, world)


def rank_rows(rows: int, world: int, rank: int) -> Tuple[int, int]:
    """[start, stop) of the real (unpadded) rows rank ``rank`` owns."""
    rpr = padded_rows(rows, world) // world
    start = min(rank * rpr, rows)
    return start, min(start + rpr, rows)

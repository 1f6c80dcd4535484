"""Data-parallel serving across the GPUs of one box with hot-replicated / cold-sharded item KV
(§5.2, Algorithm 1) — host orchestration over the C ABI.

One process per GPU (torch.distributed for the bootstrap only).  Every rank holds a full
weight replica and serves its own requests (requests are independent, so there
is no per-layer collective).  Items are placed by Algorithm 1 (bat_hrcs_place): the hottest
r·|F| items are replicated on every rank, the rest are owned round-robin by hotness rank.
Before a batch, each rank pulls the cold items it needs but does not own from the owners'
pools over NVLink (CUDA-IPC-mapped arenas, one page-copy kernel: bat_kv_fetch).

The collective steps here are bootstrap only: all_gather of the pools' IPC handles and of
the owners' page tables.  Works with the "gloo" backend and index-only pools (device = -1)
for CPU tests of the host logic.
"""
from __future__ import annotations

from typing import Dict, Iterable, List, Sequence, Tuple

import numpy as np

from . import bat


def place_items(freq: Sequence[float], r_max: float, world: int) -> Tuple[float, np.ndarray]:
    """Algorithm 1 lines 8-18: (replication ratio r, owner[i] = -1 replicated else rank)."""
    return bat.bat_hrcs_place(freq, r_max, world)


def rmax_for_nvlink(link_gbs: float, t_request_s: float, alpha: float, c: int, tau_i: float,
                    world: int, kv_bytes_per_token: int) -> float:
    """Algorithm 1 lines 4-7 with B = NVLink bandwidth converted to tokens/s."""
    B_tok = link_gbs * 1e9 / kv_bytes_per_token
    return bat.bat_hrcs_rmax(B_tok, t_request_s, alpha, c, tau_i, world)


def local_items(owner: np.ndarray, rank: int) -> List[int]:
    """Items whose KV this rank stores: the replicated ones and the ones it owns."""
    return [int(i) for i in np.nonzero((owner < 0) | (owner == rank))[0]]


def exchange_remote(pool: int, owner: np.ndarray, rank: int, world: int, group=None,
                    attach_ipc: bool = True) -> int:
    """Bootstrap collective: all_gather the pools' IPC handles (attach every peer arena) and the
    page tables of each rank's owned items; register the other ranks' items as remote entries.
    Returns the number of remote entries registered."""
    import torch.distributed as dist
    if attach_ipc:
        handles: List = [None] * world
        dist.all_gather_object(handles, bat.bat_pool_ipc_handle(pool), group=group)
        for r in range(world):
            if r != rank:
                bat.bat_pool_attach_peer(pool, r, handles[r])
    mine: Dict[int, Tuple[int, List[int]]] = {}
    for i in np.nonzero(owner == rank)[0]:
        n_tok, pages = bat.bat_kv_lookup(pool, bat.BAT_ENT_ITEM, int(i))
        mine[int(i)] = (n_tok, [int(p) for p in pages])
    tables: List = [None] * world
    dist.all_gather_object(tables, mine, group=group)
    n = 0
    for r in range(world):
        if r == rank:
            continue
        for i, (n_tok, pages) in tables[r].items():
            bat.bat_kv_register_remote(pool, bat.BAT_ENT_ITEM, int(i), r, pages, n_tok)
            n += 1
    return n


def cold_items(queries: Iterable, owner: np.ndarray, rank: int) -> np.ndarray:
    """Deduplicated ids of the items a batch needs that live on other ranks (IP requests only:
    UP requests carry their items in the suffix)."""
    need = set()
    for q in queries:
        if q.use_cache and q.order == "IP":
            for i in q.item_ids:
                o = owner[int(i)]
                if o >= 0 and o != rank:
                    need.add(int(i))
    return np.array(sorted(need), dtype=np.int64)


def fetch_cold(pool: int, ids: np.ndarray, stream=None) -> int:
    """Pull the cold items over NVLink into local pages (bat_kv_fetch); returns entries pulled."""
    if len(ids) == 0:
        return 0
    return bat.bat_kv_fetch(pool, bat.BAT_ENT_ITEM, ids, stream)


def drop_fetched(pool: int, ids: np.ndarray) -> None:
    """Release the local copies of pulled items (a per-batch staging policy)."""
    for i in ids:
        bat.bat_kv_evict(pool, bat.BAT_ENT_ITEM, int(i))


def partition_requests(lengths: Sequence[int], world: int) -> List[List[int]]:
    """Greedy load balance of requests over ranks by suffix tokens, longest first (the paper's
    "load-balanced manner").  Returns the request indices of every rank."""
    order = sorted(range(len(lengths)), key=lambda i: (-lengths[i], i))
    load = [0] * world
    out: List[List[int]] = [[] for _ in range(world)]
    for i in order:
        r = min(range(world), key=lambda k: (load[k], k))
        out[r].append(i)
        load[r] += lengths[i]
    return [sorted(x) for x in out]

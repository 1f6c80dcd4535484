"""Data-parallel serving across the GPUs of one box with hot-replicated / cold-sharded item KV
(§5.2, Algorithm 1) — host orchestration over the C ABI.

One process per GPU (torch.distributed for the bootstrap only).  Every rank holds a full
weight replica and serves its own requests (requests are independent, so there
is no per-layer collective).  Items are placed by Algorithm 1 (bat_hrcs_place): the hottest
r·|F| items are replicated on every rank, the rest are owned round-robin by hotness rank.
Before a batch, each rank pulls the cold items it needs but does not own from the owners'
pools over NVLink (CUDA-IPC-mapped arenas) with copy engines on a dedicated copy stream, one batch
ahead of the compute: ``ColdPipeline`` (reference-counted bat_kv_fetch / stream-ordered
bat_kv_release) for batches planned at call time, or staged pre-built plans (bat_plan_build_staged
/ bat_plan_fetch, double-buffered slots) for the device-resident bench leg.  Requests are routed
with user affinity for User-as-prefix requests and suffix-token balancing (``route_requests``).

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
    """Pull the cold items over NVLink into local pages (bat_kv_fetch on `stream`, copy engines;
    reference counted); returns entries copied."""
    if len(ids) == 0:
        return 0
    return bat.bat_kv_fetch(pool, bat.BAT_ENT_ITEM, ids, stream)


def release_cold(pool: int, ids: np.ndarray, stream=None) -> None:
    """Drop this batch's references to its pulled items; pages freed in `stream` order."""
    if len(ids):
        bat.bat_kv_release(pool, bat.BAT_ENT_ITEM, ids, stream)


def drop_fetched(pool: int, ids: np.ndarray) -> None:
    """Evict the local copies of pulled items outright (host-ordered; no work may still read them)."""
    for i in ids:
        bat.bat_kv_evict(pool, bat.BAT_ENT_ITEM, int(i))


class ColdPipeline:
    """One-batch-ahead cold-item pulls on a dedicated copy stream (fetched from peer GPUs
    "overlapped with compute").  ``prefetch(k, ids)`` enqueues batch k's pulls on the copy stream and
    records an event; ``acquire(k)`` makes the compute stream wait for it; ``release(k)`` drops the
    batch's references in compute-stream order after its work is enqueued.  Per step:
    acquire(k), enqueue batch k's compute, prefetch(k + 1) (its copies run under batch k's
    compute; items batch k also holds only gain a reference), release(k).  torch streams/events are
    plumbing only; the copies are libbat's (bat_kv_fetch / bat_kv_release)."""

    def __init__(self, pool: int, compute_stream, copy_stream):
        import torch
        self.torch = torch
        self.pool, self.compute, self.copy = pool, compute_stream, copy_stream
        self.ready: Dict[int, object] = {}
        self.ids: Dict[int, np.ndarray] = {}
        self.pulled = 0

    def prefetch(self, k: int, ids: np.ndarray) -> None:
        ev = self.torch.cuda.Event()
        self.pulled += fetch_cold(self.pool, ids, self.copy)
        ev.record(self.copy)
        self.ready[k], self.ids[k] = ev, ids

    def acquire(self, k: int) -> None:
        self.compute.wait_event(self.ready.pop(k))

    def release(self, k: int) -> None:
        release_cold(self.pool, self.ids.pop(k), self.compute)


def measure_pull_gbs(pool: int, peer: int, peer_pages: Sequence[int], page_bytes: int, stream, reps: int = 3) -> float:
    """Measured peer -> local pull bandwidth (GB/s) through the production pull path: the peer's
    pages are registered as temporary remote items (ids < 0), pulled with bat_kv_fetch on
    `stream` and timed with CUDA events, then released.  Feeds Algorithm 1's B."""
    import torch
    ids = np.array([-1000 - i for i in range(len(peer_pages))], dtype=np.int64)
    for i, pg in zip(ids, peer_pages):
        bat.bat_kv_register_remote(pool, bat.BAT_ENT_ITEM, int(i), peer, [int(pg)], 16)
    best = 0.0
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        fetch_cold(pool, ids, stream)
        e1.record(stream)
        e1.synchronize()
        release_cold(pool, ids, stream)
        ms = e0.elapsed_time(e1)
        best = max(best, len(ids) * page_bytes / (ms / 1e3) / 1e9)
    torch.cuda.current_stream().synchronize()
    stream.synchronize()
    return best


def route_requests(queries: Sequence, world: int, user_rank=None) -> List[List[int]]:
    """Route a global batch over the ranks ("load-balanced manner"): a cached
    User-as-prefix request goes to the rank holding its user's prefix (user affinity, default
    user_id mod world); the other requests fill the least-loaded rank by suffix tokens, longest
    first.  Returns the request indices of every rank."""
    user_rank = user_rank or (lambda uid: int(uid) % world)
    def suffix(q):
        items = sum(len(t) for t in q.item_toks)
        if not q.use_cache:
            return len(q.user_tok) + items + len(q.instr_tok) + len(q.header_tok)
        return (items if q.order == "UP" else len(q.user_tok)) + len(q.instr_tok)
    out: List[List[int]] = [[] for _ in range(world)]
    load = [0] * world
    rest = []
    for i, q in enumerate(queries):
        if q.use_cache and q.order == "UP":
            r = user_rank(q.user_id)
            out[r].append(i)
            load[r] += suffix(q)
        else:
            rest.append(i)
    for i in sorted(rest, key=lambda i: (-suffix(queries[i]), i)):
        r = min(range(world), key=lambda k: (load[k], k))
        out[r].append(i)
        load[r] += suffix(queries[i])
    return [sorted(x) for x in out]


def refresh_placement(owner_old: Sequence[int], freq_new: Sequence[float], r: float, world: int) -> np.ndarray:
    """Background placement update (P:312 Step 3, footnote P:322): bat_hrcs_refresh."""
    return bat.bat_hrcs_refresh(owner_old, freq_new, r, world)


def apply_refresh(pool: int, model: int, owner_old: Sequence[int], owner_new: Sequence[int], rank: int,
                  token_fn, pos0: int = 0, stream=None) -> Dict[str, int]:
    """Apply a placement refresh on this rank's pool: items promoted into the replicated area are
    pulled from their owner as regular local entries (bat_kv_replicate), items demoted from it
    are dropped unless this rank is their new owner (bat_kv_evict), and new items this rank
    stores (owned or replicated) are computed by the prefix-miss path (bat_kv_prefill_entities;
    token_fn(id) gives an item's tokens).  Afterwards every rank calls exchange_remote with
    owner_new so the remote tables name the new owners.  Returns the move counts."""
    import torch
    n_old = len(owner_old)
    promote = [i for i in range(n_old) if owner_old[i] >= 0 and owner_new[i] < 0 and owner_old[i] != rank]
    drop = [i for i in range(n_old) if owner_old[i] < 0 and owner_new[i] >= 0 and owner_new[i] != rank]
    new = [i for i in range(n_old, len(owner_new)) if owner_new[i] < 0 or owner_new[i] == rank]
    if promote:
        bat.bat_kv_replicate(pool, bat.BAT_ENT_ITEM, promote, stream)
    torch.cuda.synchronize()  # background refresh: nothing may still read the dropped pages
    for i in drop:
        bat.bat_kv_evict(pool, bat.BAT_ENT_ITEM, int(i))
    for s in range(0, len(new), 256):
        ids = new[s:s + 256]
        bat.bat_kv_prefill_entities(pool, model, bat.BAT_ENT_ITEM, ids, [token_fn(i) for i in ids], pos0, stream=stream)
    return dict(promoted=len(promote), dropped=len(drop), computed=len(new))


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

"""Device-memory helpers around the C ABI (PyTorch used only for memory and streams).

``DeviceModel`` uploads a weight set to bf16 device tensors in the layout of include/bat.h
and owns the ``bat_model`` handle; ``DevicePool`` owns a ``bat_pool``.  Neither computes any
step of the method.
"""
from __future__ import annotations

from typing import Dict, List, Optional

import numpy as np

from . import bat

LAYER_KEYS = ("ln1", "wqkv", "bqkv", "wo", "ln2", "wgu", "wd")


def _torch():
    import torch
    return torch


class DeviceModel:
    """Weights (bf16 device tensors; dtype="fp32" for the SIMT correctness mode) + the
    library's model handle.

    ``source`` is any object with ``cfg`` (dict), ``embed_full()``, ``lm_head_full()``,
    ``final_norm()`` and ``layer(l)`` returning the 7 per-layer arrays, or
    ``tensors=`` a dict {"embed", "lm_head" (optional: tied), "final_norm", "layers": [...]}
    of device tensors already in bf16."""

    def __init__(self, cfg: dict, source=None, tensors: Optional[dict] = None, device: int = 0,
                 dtype: str = "bf16"):
        torch = _torch()
        self.cfg = dict(cfg)
        self.device = device
        self.dtype = dtype
        dev = torch.device("cuda", device)
        tdt = {"bf16": torch.bfloat16, "fp32": torch.float32}[dtype]  # fp32: SIMT correctness mode
        to = lambda a: torch.as_tensor(np.asarray(a, dtype=np.float32)).to(dev, tdt).contiguous()
        if tensors is None:
            embed = to(source.embed_full())
            lm = embed if cfg.get("tied") else to(source.lm_head_full())
            fin = to(source.final_norm())
            layers = []
            for l in range(cfg["layers"]):
                w = source.layer(l)
                layers.append({k: to(w[k]) for k in LAYER_KEYS})
            tensors = dict(embed=embed, lm_head=lm, final_norm=fin, layers=layers)
        if tensors.get("lm_head") is None:
            tensors["lm_head"] = tensors["embed"]
        self.t = tensors
        ptrs = [tensors["embed"].data_ptr(), tensors["lm_head"].data_ptr(), tensors["final_norm"].data_ptr()]
        for lw in tensors["layers"]:
            ptrs += [lw[k].data_ptr() for k in LAYER_KEYS]
        self.handle = bat.bat_model_create(cfg, ptrs, device,
                                           bat.BAT_FP32 if dtype == "fp32" else bat.BAT_BF16)

    def close(self):
        if self.handle:
            bat.bat_model_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class DevicePool:
    def __init__(self, cfg: dict, num_pages: int, device: int = 0, rank: int = 0, world: int = 1,
                 dtype: str = "bf16"):
        self.cfg = dict(cfg)
        self.device = device
        self.handle = bat.bat_kv_pool_create(device, num_pages, cfg["layers"], cfg["kv_heads"],
                                             cfg["head_dim"], bat.BAT_FP32 if dtype == "fp32" else bat.BAT_BF16,
                                             rank=rank, world=world)

    def close(self):
        if self.handle:
            bat.bat_kv_pool_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def needed_entities(queries) -> Dict[tuple, np.ndarray]:
    """The (kind, id) -> tokens of every prefix entry a batch of cached requests needs
    (UP: the user; IP: header + items) — bookkeeping only."""
    out: Dict[tuple, np.ndarray] = {}
    for q in queries:
        if not q.use_cache:
            continue
        if q.order == "UP":
            out[(bat.BAT_ENT_USER, int(q.user_id))] = np.asarray(q.user_tok, np.int32)
        else:
            if len(q.header_tok):
                out[(bat.BAT_ENT_HEADER, int(q.header_id))] = np.asarray(q.header_tok, np.int32)
            for iid, t in zip(q.item_ids, q.item_toks):
                out[(bat.BAT_ENT_ITEM, int(iid))] = np.asarray(t, np.int32)
    return out


def prefill_missing_entities(pool: DevicePool, model: DeviceModel, queries, stream=None,
                             batch: int = 256) -> int:
    """Compute and cache every prefix entry the batch needs that the pool lacks (the
    prefix-miss path), through bat_kv_prefill_entities.  Returns the count."""
    ents = needed_entities(queries)
    n = 0
    headers = {k: v for k, v in ents.items() if k[0] == bat.BAT_ENT_HEADER}
    for (kind, eid), toks in headers.items():
        try:
            bat.bat_kv_lookup(pool.handle, kind, eid)
            continue
        except bat.BatError:
            pass
        bat.bat_kv_prefill_entities(pool.handle, model.handle, kind, [eid], [toks], 0, stream=stream)
        n += 1
    # an item's KV is computed in the context its requests give it: after their header (reading
    # R3) or alone; the context of every item is the header id of the IP requests using it
    item_ctx: Dict[int, int] = {}
    hdr_len: Dict[int, int] = {}
    for q in queries:
        if not (q.use_cache and q.order == "IP"):
            continue
        h = int(q.header_id) if len(q.header_tok) else -1
        if h >= 0:
            hdr_len[h] = len(q.header_tok)
        for iid in q.item_ids:
            prev = item_ctx.setdefault(int(iid), h)
            if prev != h:
                raise ValueError(f"item {int(iid)} is used after different headers in one batch")
    for kind in (bat.BAT_ENT_USER, bat.BAT_ENT_ITEM):
        todo = []
        for (k, eid), toks in ents.items():
            if k != kind:
                continue
            try:
                bat.bat_kv_lookup(pool.handle, kind, eid)
            except bat.BatError:
                todo.append((eid, toks))
        groups: Dict[int, List] = {}
        for eid, toks in todo:
            groups.setdefault(item_ctx.get(int(eid), -1) if kind == bat.BAT_ENT_ITEM else -1, []).append((eid, toks))
        for hid, lst in groups.items():
            for s in range(0, len(lst), batch):
                chunk = lst[s:s + batch]
                if hid >= 0:
                    bat.bat_kv_prefill_entities(pool.handle, model.handle, kind, [e for e, _ in chunk],
                                                [t for _, t in chunk], hdr_len[hid], bat.BAT_ENT_HEADER, hid, stream)
                else:
                    bat.bat_kv_prefill_entities(pool.handle, model.handle, kind, [e for e, _ in chunk],
                                                [t for _, t in chunk], 0, stream=stream)
                n += len(chunk)
    return n


class TraceServer:
    """The serving loop of P:288-294 on one GPU: the prompt scheduler
    (bat_sched_*: P:366 / P:377 prefix selection over the user-prefix cache index) decides each
    request's prefix side in arrival order; its cache actions are applied to the pool (evicted
    users -> bat_kv_evict, admitted users -> their prefix KV computed by the prefix-miss path);
    batches run through bat_bipartite_prefill + bat_score.  Bookkeeping only — every step of the
    method runs in libbat."""

    def __init__(self, pool: DevicePool, model: DeviceModel, policy: str, user_capacity_pages: int,
                 window: float, seed: int = 0, n_instr: int = 8, item_len=(16, 16)):
        self.pool, self.model, self.cfg = pool, model, model.cfg
        self.sched = bat.bat_sched_create(policy, user_capacity_pages, window)
        self.seed, self.n_instr, self.item_len = seed, n_instr, item_len
        self.decisions = []

    def close(self):
        if self.sched:
            bat.bat_sched_destroy(self.sched)
            self.sched = None

    def _run(self, pending, k, out):
        if not pending:
            return
        torch = _torch()
        prefill_missing_entities(self.pool, self.model, pending)
        dev = torch.device("cuda", self.model.device)
        Bn = len(pending)
        n_max = max(q.n_items for q in pending)
        hidden = torch.empty(Bn, self.cfg["hidden"], device=dev)
        bat.bat_bipartite_prefill(self.pool.handle, self.model.handle, bat.QueryArray(pending), hidden)
        labels = np.zeros((Bn, n_max), np.int32)
        for b, q in enumerate(pending):
            labels[b, : q.n_items] = q.labels
        scores = torch.empty(Bn, n_max, device=dev)
        topk = torch.empty(Bn, max(k, 1), dtype=torch.int32, device=dev)
        bat.bat_score(self.model.handle, hidden, torch.tensor(labels, device=dev),
                      torch.tensor([q.n_items for q in pending], dtype=torch.int32, device=dev), Bn, n_max,
                      scores, k, topk if k else None)
        out.append((list(pending), hidden, scores))
        pending.clear()

    def serve(self, requests, batch: int = 16, k: int = 0):
        """requests: iterable of (time, user_id, n_user_tokens, item_ids).  Returns a list of
        (queries, hidden [B][H], scores [B][n_max]) per executed batch, in order."""
        import synth
        out, pending, pinned = [], [], set()
        for (t, uid, n_user, item_ids) in requests:
            tau_i = sum(synth.item_length(int(i), *self.item_len, self.seed) for i in item_ids)
            order, hit, admit, evicted, f = bat.bat_sched_decide(self.sched, t, uid, n_user, tau_i)
            if any(e in pinned for e in evicted):  # a queued UP request still needs that user
                self._run(pending, k, out)
                pinned.clear()
            for e in evicted:
                try:
                    bat.bat_kv_evict(self.pool.handle, bat.BAT_ENT_USER, e)
                except bat.BatError:
                    pass  # admitted but never materialised (its batch had not run)
            q = synth.make_query(self.seed, self.cfg, uid, n_user, item_ids, self.item_len, self.n_instr,
                                 "UP" if order == "UP" else "IP", use_cache=(order != "RE"))
            if order == "UP" and not admit and not hit:
                q.use_cache = False  # UP-only baseline with a user larger than the cache
            if order == "UP" and q.use_cache:
                pinned.add(uid)
            self.decisions.append((order, hit, admit, evicted))
            pending.append(q)
            if len(pending) == batch:
                self._run(pending, k, out)
                pinned.clear()
        self._run(pending, k, out)
        return out

    def stats(self) -> dict:
        return bat.bat_sched_stats(self.sched)

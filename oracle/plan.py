"""The integer plan of one batch, by brute force (TEST INFRASTRUCTURE ONLY).

What it computes (SURVEY §8(c) "Plan definition"; DESIGN.md §"Plan"):

* per query, the suffix tokens in prompt order with their positions and segment ids
  (P:249-257 via oracle.sequence.build_sequence) — the prefix side is UP: the user
  entity; IP: [header entity] + the items in candidate order; RE (use_cache=0): nothing;
* the query's key slots: every prefix entity's pages (entries at user/item
  granularity, paged, each entity starting on a fresh page of 16 slots), then the suffix
  keys, page-padded; key metadata kseg (segment) and kord (0 for a prefix key, suffix
  index + 1 for a suffix key, INVALID for an empty slot);
* row metadata rseg, rord (suffix index + 1);
* the tile-state matrix: q-tile i (rows = tokens [i*qt, (i+1)*qt) x the g heads of one KV
  head) against k-tile j (key slots [128 j, 128 j + 128)): 0 = no visible pair, 1 = every
  pair visible, 2 = some.  Visibility (reading R4/R5/R6):
      kord[k] <= rord[t]  and  (kseg[k] == rseg[t] or kseg[k] < 0 or rseg[t] < 0).
  Computed here by enumerating every pair.
"""
from __future__ import annotations

from typing import Dict, List, Sequence, Tuple

import numpy as np

from .sequence import build_sequence

PAGE = 16
KTILE_PAGES = 8
KTILE = PAGE * KTILE_PAGES
INVALID_ORD = 2 ** 31 - 1
ENT_USER, ENT_ITEM, ENT_HEADER = 0, 1, 2
USER_SEG, INSTR_SEG, HEADER_SEG = -1, -2, -3


def qtile_tokens(group: int, rows: int = 128) -> int:
    """Tokens per packed q-tile: rows = tokens x group heads of one KV head."""
    return rows // group


def prefix_entities(q) -> List[Tuple[int, int, int]]:
    """[(kind, id, seg)] of the query's prefix, in prompt order."""
    if not q.use_cache:
        return []
    if q.order == "UP":
        return [(ENT_USER, int(q.user_id), USER_SEG)]
    ents = []
    if len(q.header_tok):
        ents.append((ENT_HEADER, int(q.header_id), HEADER_SEG))
    for i, iid in enumerate(q.item_ids):
        ents.append((ENT_ITEM, int(iid), i))
    return ents


def plan_query(q, entity_pages: Dict[Tuple[int, int], Tuple[Sequence[int], int]],
               group: int, scratch_page0: int = 0) -> dict:
    pic = int(getattr(q, "pic_tail", 0) or 0) if q.order == "IP" else 0
    tokens, seg, pos = build_sequence(q.order, q.user_tok, q.item_toks, q.instr_tok,
                                      q.header_tok if q.order == "IP" else (), pic)

    def used(kind, eid):  # prefix tokens served from an entry: an item's head under PIC (R25)
        n = entity_pages[(kind, eid)][1]
        return n - min(pic, n) if kind == ENT_ITEM else n

    ents = prefix_entities(q)
    P = sum(used(k, i) for (k, i, _) in ents)
    S = len(tokens) - P
    pages: List[int] = []
    valid: List[int] = []
    kseg: List[int] = []
    kord: List[int] = []
    for (kind, eid, sg) in ents:
        plist, n_all = entity_pages[(kind, eid)]
        assert len(plist) == (n_all + PAGE - 1) // PAGE
        n = used(kind, eid)
        plist = plist[: (n + PAGE - 1) // PAGE]
        for pi, p in enumerate(plist):
            nv = min(PAGE, n - pi * PAGE)
            pages.append(int(p))
            valid.append(nv)
            for j in range(PAGE):
                kseg.append(sg if j < nv else -1)
                kord.append(0 if j < nv else INVALID_ORD)
    n_pre = len(pages)
    n_sfx_pages = (S + PAGE - 1) // PAGE
    for sp in range(n_sfx_pages):
        nv = min(PAGE, S - sp * PAGE)
        pages.append(-(scratch_page0 + sp) - 1)  # scratch page s encoded as -(s+1)
        valid.append(nv)
        for j in range(PAGE):
            t = sp * PAGE + j
            kseg.append(int(seg[P + t]) if j < nv else -1)
            kord.append(t + 1 if j < nv else INVALID_ORD)
    rseg = seg[P:].astype(np.int64)
    rord = np.arange(1, S + 1, dtype=np.int64)
    kseg_a = np.array(kseg, dtype=np.int64)
    kord_a = np.array(kord, dtype=np.int64)

    # brute-force visibility over every (row, key-slot) pair
    vis = (kord_a[None, :] <= rord[:, None]) & (
        (kseg_a[None, :] == rseg[:, None]) | (kseg_a[None, :] < 0) | (rseg[:, None] < 0))
    qt = qtile_tokens(group)
    n_qt = (S + qt - 1) // qt
    n_kslots = len(kseg)
    n_kt = (n_kslots + KTILE - 1) // KTILE
    state = np.zeros((n_qt, n_kt), dtype=np.int64)
    for i in range(n_qt):
        r0, r1 = i * qt, min(S, (i + 1) * qt)
        for j in range(n_kt):
            k0, k1 = j * KTILE, (j + 1) * KTILE
            blk = vis[r0:r1, k0:min(k1, n_kslots)]
            n_live = int(blk.sum())
            full_pairs = (r1 - r0) * KTILE  # slots past the last page are empty (invalid)
            state[i, j] = 0 if n_live == 0 else (1 if n_live == full_pairs else 2)
    # discriminant suffix rows: the last token or, with one discriminant per item
    # (reading R20), the last token of every item, in candidate order
    if getattr(q, "multi_disc", False):
        disc = np.array([int(np.nonzero(rseg == i)[0].max()) for i in range(len(q.item_toks))], dtype=np.int64)
    else:
        disc = np.array([S - 1], dtype=np.int64)
    return dict(tokens=tokens[P:].astype(np.int64), pos=pos[P:].astype(np.int64), disc=disc,
                seg=rseg, P=P, S=S, pages=np.array(pages, dtype=np.int64),
                valid=np.array(valid, dtype=np.int64), n_prefix_pages=n_pre,
                kseg=kseg_a, kord=kord_a, rord=rord, tile_state=state, vis=vis,
                n_live_pairs=int(vis.sum()))


def plan_batch(queries, entity_pages, group: int) -> List[dict]:
    out, sp, tok0 = [], 0, 0
    for q in queries:
        p = plan_query(q, entity_pages, group, sp)
        p["scratch_page0"] = sp
        p["token_off"] = tok0
        sp += (p["S"] + PAGE - 1) // PAGE
        tok0 += p["S"]
        out.append(p)
    return out

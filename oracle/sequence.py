"""Prompt ordering, segments, bipartite positions and the explicit mask.

PAPER.md P:249 (User-as-prefix order [U, I_1..I_N, Instr]), P:253 (Item-as-prefix order
[I_1..I_N, U, Instr]), P:257 ("Attention Masks and Position Encoding": items cannot attend
to each other, all items share the same starting position id: |U| in UP, 0 — or after
notation tokens — in IP), P:131 (Fig. 1: "The attention across different items is masked
out").  Readings (R2, R3, R5): positions after the item set continue from the
maximum item length m; header tokens precede the items in IP; attention is causal within
every segment.
"""
from __future__ import annotations

import numpy as np

USER = -1
INSTR = -2
HEADER = -3


def build_sequence(order: str, user_tok, item_toks, instr_tok, header_tok=(), pic_tail: int = 0):
    """Return (tokens, seg, pos) of the full prompt as int64 arrays.

    seg: USER / INSTR / HEADER, or the candidate index i >= 0 for item tokens.
    pos: UP  — U: 0..|U|-1; item i token j: |U| + j; Instr k: |U| + m + k
         IP  — header: 0..h-1; item i token j: h + j; U token p: h + m + p;
               Instr k: h + m + |U| + k
    where m = max_i |I_i| (reading R2) and h = len(header_tok) (reading R3, IP only).

    pic_tail = k > 0 (IP only; selective recompute, P:265 / P:476, reading R25): the last
    k_i = min(k, |I_i|) tokens of every item move after U — order [header, item heads, U,
    item tails (candidate order), Instr] — at positions h + m + |U| + j for item token j, and
    Instr continues at h + m + |U| + m + k'; item heads keep h + j.  k = 0 is plain IP.
    """
    user_tok = np.asarray(user_tok, dtype=np.int64)
    instr_tok = np.asarray(instr_tok, dtype=np.int64)
    header_tok = np.asarray(header_tok, dtype=np.int64)
    items = [np.asarray(t, dtype=np.int64) for t in item_toks]
    m = max((len(t) for t in items), default=0)
    nu, nx = len(user_tok), len(instr_tok)
    toks, segs, poss = [], [], []

    def put(t, s, p):
        toks.append(np.asarray(t, dtype=np.int64))
        segs.append(np.full(len(t), s, dtype=np.int64) if np.isscalar(s) else np.asarray(s))
        poss.append(np.asarray(p, dtype=np.int64))

    if order == "UP":
        if len(header_tok):
            raise ValueError("header tokens are an Item-as-prefix notion (P:257)")
        put(user_tok, USER, np.arange(nu))
        for i, t in enumerate(items):
            put(t, i, nu + np.arange(len(t)))
        put(instr_tok, INSTR, nu + m + np.arange(nx))
    elif order == "IP":
        h = len(header_tok)
        put(header_tok, HEADER, np.arange(h))
        tails = [min(int(pic_tail), len(t)) for t in items]
        for i, t in enumerate(items):                 # cached heads (all of every item when k = 0)
            put(t[: len(t) - tails[i]], i, h + np.arange(len(t) - tails[i]))
        put(user_tok, USER, h + m + np.arange(nu))
        for i, t in enumerate(items):                 # recomputed tails, after U
            put(t[len(t) - tails[i]:], i, h + m + nu + np.arange(len(t) - tails[i], len(t)))
        x0 = h + m + nu + (m if sum(tails) > 0 else 0)
        put(instr_tok, INSTR, x0 + np.arange(nx))
    else:
        raise ValueError(order)
    return np.concatenate(toks), np.concatenate(segs), np.concatenate(poss)


def visible(seg_q, idx_q, seg_k, idx_k) -> bool:
    """Scalar visibility: causal in sequence order and not (two different items)."""
    if idx_k > idx_q:
        return False
    if seg_q >= 0 and seg_k >= 0 and seg_q != seg_k:
        return False
    return True


def bipartite_mask(seg) -> np.ndarray:
    """M[q, k] = (k <= q) and not (seg[q] >= 0 and seg[k] >= 0 and seg[q] != seg[k])."""
    seg = np.asarray(seg)
    T = len(seg)
    causal = np.tril(np.ones((T, T), dtype=bool))
    qi = seg[:, None]
    ki = seg[None, :]
    cross_item = (qi >= 0) & (ki >= 0) & (qi != ki)
    return causal & ~cross_item


def causal_mask(T: int) -> np.ndarray:
    return np.tril(np.ones((T, T), dtype=bool))


def prefix_length(order: str, user_tok, item_toks, header_tok=(), pic_tail: int = 0) -> int:
    """P: number of prompt tokens that are served from the prefix cache."""
    if order == "UP":
        return len(user_tok)
    return len(header_tok) + sum(len(t) - min(int(pic_tail), len(t)) for t in item_toks)

"""Qwen2-shaped GR ranking forward in fp64 (TEST INFRASTRUCTURE ONLY — see oracle/__init__).

PAPER.md §2.2: h^(0)_t = E[x_t]; L transformer layers (multi-head self-attention
followed by an FFN) give h^(L).  §3.2: with a cached prefix, only the suffix is
projected and it attends to [k_{1:P}; k_{P+1:T}].  The layer internals (RMSNorm, q/k/v with
bias, rotate-half RoPE, GQA, SwiGLU) are the public Qwen2 architecture the paper evaluates
(Table 2), not PAPER.md text; the N=1 special case is pinned against the
HuggingFace transformers Qwen2 implementation (tests/test_oracle_model.py).

Everything is float64 on bf16-exact weights (reading R10).  The attention is the
naive definition: for every head, scores of all (query, key) pairs, -inf where the explicit
boolean mask forbids, softmax, weighted sum of values.
"""
from __future__ import annotations

from typing import List, Optional, Sequence, Tuple

import numpy as np

from .sequence import bipartite_mask, build_sequence, causal_mask, HEADER, USER
from .score import score as score_fn


def rmsnorm(x: np.ndarray, g: np.ndarray, eps: float) -> np.ndarray:
    """x / sqrt(mean(x^2) + eps) * g."""
    return x / np.sqrt(np.mean(x * x, axis=-1, keepdims=True) + eps) * g


def rope(x: np.ndarray, pos: np.ndarray, theta: float) -> np.ndarray:
    """Rotate-half RoPE: pairs (i, i + d/2), inv_freq_i = theta^(-2i/d), angle = pos*inv_freq.
    x: [T, heads, d]."""
    d = x.shape[-1]
    half = d // 2
    inv_freq = theta ** (-(np.arange(half, dtype=np.float64) * 2.0) / d)
    ang = np.asarray(pos, dtype=np.float64)[:, None] * inv_freq[None, :]
    cos = np.cos(ang)[:, None, :]
    sin = np.sin(ang)[:, None, :]
    x1, x2 = x[..., :half], x[..., half:]
    return np.concatenate([x1 * cos - x2 * sin, x2 * cos + x1 * sin], axis=-1)


def silu(x: np.ndarray) -> np.ndarray:
    return x / (1.0 + np.exp(-x))


def attention(q: np.ndarray, k: np.ndarray, v: np.ndarray, mask: np.ndarray,
              group: int) -> np.ndarray:
    """o[t, j] = sum_k softmax_k(q[t,j].k[k,j//g] / sqrt(d) over {k: mask[t,k]}) v[k, j//g].

    q: [T, Hq, d]; k, v: [Tk, Hkv, d]; mask: [T, Tk] bool."""
    T, Hq, d = q.shape
    out = np.zeros((T, Hq, d), dtype=np.float64)
    scale = 1.0 / np.sqrt(d)
    for j in range(Hq):
        kv = j // group
        s = (q[:, j, :] @ k[:, kv, :].T) * scale
        s = np.where(mask, s, -np.inf)
        mx = np.max(s, axis=1, keepdims=True)
        p = np.where(mask, np.exp(s - mx), 0.0)
        p = p / np.sum(p, axis=1, keepdims=True)
        out[:, j, :] = p @ v[:, kv, :]
    return out


def layer_forward(cfg: dict, w: dict, h: np.ndarray, pos: np.ndarray,
                  k_pre: Optional[np.ndarray], v_pre: Optional[np.ndarray],
                  mask: np.ndarray, rope_on: bool = True):
    """One Qwen2 block over S rows h [S,H]; keys = [prefix keys ; the S rows' own keys];
    mask [S, P+S].  Returns (h_out, k, v) with k, v the S rows' post-RoPE keys/values."""
    H, d, Hq, Hkv, F = cfg["hidden"], cfg["head_dim"], cfg["q_heads"], cfg["kv_heads"], cfg["ffn"]
    S = h.shape[0]
    f64 = lambda a: np.asarray(a, dtype=np.float64)
    a = rmsnorm(h, f64(w["ln1"]), cfg["rms_eps"])
    qkv = a @ f64(w["wqkv"]).T + f64(w["bqkv"])
    q = qkv[:, : Hq * d].reshape(S, Hq, d)
    k = qkv[:, Hq * d: (Hq + Hkv) * d].reshape(S, Hkv, d)
    v = qkv[:, (Hq + Hkv) * d:].reshape(S, Hkv, d)
    if rope_on:
        q = rope(q, pos, cfg["rope_theta"])
        k = rope(k, pos, cfg["rope_theta"])
    if k_pre is not None and len(k_pre):
        K = np.concatenate([k_pre, k], axis=0)
        V = np.concatenate([v_pre, v], axis=0)
    else:
        K, V = k, v
    o = attention(q, K, V, mask, Hq // Hkv)
    h = h + o.reshape(S, Hq * d) @ f64(w["wo"]).T
    b = rmsnorm(h, f64(w["ln2"]), cfg["rms_eps"])
    gu = b @ f64(w["wgu"]).T
    h = h + (silu(gu[:, :F]) * gu[:, F:]) @ f64(w["wd"]).T
    return h, k, v


def forward_full(cfg: dict, W, tokens: np.ndarray, pos: np.ndarray, mask: np.ndarray,
                 rope_on: bool = True, keep_kv: bool = False):
    """Full recompute (no cache): the plain definition.  Returns (h^(L) [T,H], kv) where kv
    is a list over layers of (K [T,Hkv,d], V) if keep_kv else None."""
    h = np.asarray(W.embed_rows(tokens), dtype=np.float64)
    kvs = [] if keep_kv else None
    for l in range(cfg["layers"]):
        h, k, v = layer_forward(cfg, W.layer(l), h, pos, None, None, mask, rope_on)
        if keep_kv:
            kvs.append((k, v))
    return h, kvs


def forward_cached(cfg: dict, W, suffix_tokens: np.ndarray, suffix_pos: np.ndarray,
                   prefix_kv: Sequence[Tuple[np.ndarray, np.ndarray]], mask: np.ndarray,
                   rope_on: bool = True, keep_kv: bool = False):
    """Prefix caching: project only the suffix; at every layer l the suffix
    attends to [prefix_kv[l] ; its own keys] under mask [S, P+S]."""
    h = np.asarray(W.embed_rows(suffix_tokens), dtype=np.float64)
    kvs = [] if keep_kv else None
    for l in range(cfg["layers"]):
        kp, vp = prefix_kv[l] if prefix_kv is not None else (None, None)
        h, k, v = layer_forward(cfg, W.layer(l), h, suffix_pos, kp, vp, mask, rope_on)
        if keep_kv:
            kvs.append((k, v))
    return h, kvs


def entity_kv(cfg: dict, W, tokens: np.ndarray, pos0: int = 0, context_tokens=(),
              rope_on: bool = True):
    """Standalone KV of one cache entry (a user; an item): the entity's
    tokens run alone (after optional context tokens, e.g. the IP header) with a causal mask
    at positions pos0.. ; returns per-layer (K, V) of the entity's own tokens."""
    ctx = np.asarray(context_tokens, dtype=np.int64)
    toks = np.concatenate([ctx, np.asarray(tokens, dtype=np.int64)])
    pos = np.concatenate([np.arange(len(ctx)), pos0 + np.arange(len(tokens))])
    _, kvs = forward_full(cfg, W, toks, pos, causal_mask(len(toks)), rope_on, keep_kv=True)
    n0 = len(ctx)
    return [(k[n0:], v[n0:]) for (k, v) in kvs]


def final_hidden(cfg: dict, W, h_last: np.ndarray) -> np.ndarray:
    """hf = RMSNorm(h_T^(L); g_final)  (the discriminant token)."""
    return rmsnorm(h_last, np.asarray(W.final_norm(), dtype=np.float64), cfg["rms_eps"])


def run_query(cfg: dict, W, q, mode: str = "full", rope_on: bool = True, k: int = 0,
              mask_fn=None):
    """Serve one ranking request.

    mode "full": build the whole prompt in q.order and recompute every token (RE).
    mode "cached": the prefix side (UP: the user, IP: header + every item) is computed
    standalone per entity and reused; the suffix attends to it.
    Returns dict(hf, z, s, topk, h_last).  ``mask_fn`` overrides the bipartite mask (only
    for the mask-sensitivity guard test)."""
    tokens, seg, pos = build_sequence(q.order, q.user_tok, q.item_toks, q.instr_tok,
                                      q.header_tok if q.order == "IP" else (), _pic(q))
    mask = (mask_fn or bipartite_mask)(seg)
    if mode == "full" or not q.use_cache:
        h, _ = forward_full(cfg, W, tokens, pos, mask, rope_on)
    elif mode == "cached":
        P = _prefix_len(q)
        prefix_kv = _prefix_kv(cfg, W, q, rope_on)
        h, _ = forward_cached(cfg, W, tokens[P:], pos[P:], prefix_kv, mask[P:, :], rope_on)
    else:
        raise ValueError(mode)
    hf = final_hidden(cfg, W, h[-1])
    z, s, top = score_fn(W.lm_head_rows(q.labels), hf, k)
    return dict(hf=hf, z=z, s=s, topk=top, h_last=h[-1])


def run_query_multi(cfg: dict, W, q, mode: str = "full", rope_on: bool = True, k: int = 0):
    """Multi-discriminant variant (reading R20): in User-as-prefix order the last token of
    every item I_i is item i's discriminant; z_i = W_out[v_i] . RMSNorm(h_last(I_i)) (P:175 per
    item), s = softmax_i z_i, top-k.  Returns dict(hf [N][H], z, s, topk)."""
    assert q.order == "UP", "one discriminant per item needs the items computed (User-as-prefix)"
    tokens, seg, pos = build_sequence(q.order, q.user_tok, q.item_toks, q.instr_tok, ())
    mask = bipartite_mask(seg)
    if mode == "full" or not q.use_cache:
        h, _ = forward_full(cfg, W, tokens, pos, mask, rope_on)
        off = 0
    elif mode == "cached":
        P = _prefix_len(q)
        h, _ = forward_cached(cfg, W, tokens[P:], pos[P:], _prefix_kv(cfg, W, q, rope_on), mask[P:, :], rope_on)
        off = P
    else:
        raise ValueError(mode)
    seg = np.asarray(seg)
    rows = [int(np.nonzero(seg == i)[0].max()) - off for i in range(len(q.item_toks))]
    hf = np.stack([final_hidden(cfg, W, h[r]) for r in rows])
    Wl = np.asarray(W.lm_head_rows(q.labels), np.float64)
    z = np.einsum("ij,ij->i", Wl, hf)
    s = np.exp(z - z.max())
    s = s / s.sum()
    order = sorted(range(len(s)), key=lambda i: (-s[i], i))[:k]
    return dict(hf=hf, z=z, s=s, topk=np.asarray(order, np.int64))


def _pic(q) -> int:
    """Selective-recompute tail length of an IP request (reading R25; 0 = plain IP)."""
    return int(getattr(q, "pic_tail", 0) or 0) if q.order == "IP" else 0


def _prefix_len(q) -> int:
    if q.order == "UP":
        return len(q.user_tok)
    k = _pic(q)
    return len(q.header_tok) + sum(len(t) - min(k, len(t)) for t in q.item_toks)


def _prefix_kv(cfg: dict, W, q, rope_on: bool = True):
    """Concatenate the standalone KV of the prefix entities in prompt order."""
    if q.order == "UP":
        return entity_kv(cfg, W, q.user_tok, 0, (), rope_on)
    hdr = np.asarray(q.header_tok, dtype=np.int64)
    parts = []
    if len(hdr):
        parts.append(entity_kv(cfg, W, hdr, 0, (), rope_on))
    k = _pic(q)
    for t in q.item_toks:
        # the cached head of an item = the first |I| - k rows of its standalone KV (causal)
        kv = entity_kv(cfg, W, t, len(hdr), hdr, rope_on)
        n = len(t) - min(k, len(t))
        parts.append([(kk[:n], vv[:n]) for kk, vv in kv])
    L = cfg["layers"]
    return [(np.concatenate([p[l][0] for p in parts]), np.concatenate([p[l][1] for p in parts]))
            for l in range(L)]

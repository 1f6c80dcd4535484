"""Helpers shared by the GPU tests (marshalling and reference assembly only)."""
from __future__ import annotations

import numpy as np

import synth
from oracle import model as om
from oracle.sequence import bipartite_mask, build_sequence


def tol_ok(got, ref, atol=2e-2, rtol=2e-2):
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    return np.all(np.abs(got - ref) <= atol + rtol * np.abs(ref))


def max_excess(got, ref, atol=2e-2, rtol=2e-2):
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    return float(np.max(np.abs(got - ref) - (atol + rtol * np.abs(ref))))


def score_excess(z_gpu, s_gpu, z_ref, s_ref, atol=2e-2, rtol=2e-2):
    """Parity of the score kernel's own outputs (a9): the logits z elementwise at the north_star
    tolerance, and the scores s on a RELATIVE scale — |log s_gpu - log s_ref| within twice the
    largest logit tolerance (the bound an in-tolerance z implies for log-softmax), so that s ~ 1/N
    cannot hide behind the absolute tolerance.  Returns the worst excess of each (<= 0 passes)."""
    z_gpu, s_gpu = np.asarray(z_gpu, np.float64), np.asarray(s_gpu, np.float64)
    z_ref, s_ref = np.asarray(z_ref, np.float64), np.asarray(s_ref, np.float64)
    ez = max_excess(z_gpu, z_ref, atol, rtol)
    bound = 2.0 * float(np.max(atol + rtol * np.abs(z_ref)))
    with np.errstate(divide="ignore"):
        dl = np.abs(np.log(np.maximum(s_gpu, 1e-300)) - np.log(s_ref))
    els = float(np.max(dl) - bound)
    return ez, els


def prefix_entities_in_order(q):
    """(kind, id, tokens) of the prefix entries of a cached request, in prompt order."""
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
    if not q.use_cache:
        return []
    if q.order == "UP":
        return [(bat.BAT_ENT_USER, int(q.user_id), q.user_tok)]
    out = []
    if len(q.header_tok):
        out.append((bat.BAT_ENT_HEADER, int(q.header_id), q.header_tok))
    out += [(bat.BAT_ENT_ITEM, int(i), t) for i, t in zip(q.item_ids, q.item_toks)]
    return out


def oracle_attention_layer(cfg, q, entity_kv, qkv_rows, layer, rope_on=True, round_qk=False):
    """fp64 reference of one layer of bipartite attention for request q given the cached
    prefix K/V (entity_kv[(kind,id)] = (K [L][n][Hkv][d], V)) and the suffix's raw qkv rows.
    round_qk: round the RoPE'd suffix q and k to bf16 (RNE) — the tensor-core operands' own input
    rounding — for a TIGHTER secondary check that isolates the kernel from that rounding."""
    d, Hq, Hkv = cfg["head_dim"], cfg["q_heads"], cfg["kv_heads"]
    pic = int(getattr(q, "pic_tail", 0) or 0) if q.order == "IP" else 0
    toks, seg, pos = build_sequence(q.order, q.user_tok, q.item_toks, q.instr_tok,
                                    q.header_tok if q.order == "IP" else (), pic)
    ents = prefix_entities_in_order(q)
    # under PIC (reading R25) an item serves only its head from the cache
    used = {(k, i): (len(t) - min(pic, len(t)) if k == 1 else len(t)) for k, i, t in ents}
    P = sum(used.values())
    S = len(toks) - P
    x = np.asarray(qkv_rows, np.float64)
    assert x.shape[0] == S
    qq = x[:, : Hq * d].reshape(S, Hq, d)
    kk = x[:, Hq * d:(Hq + Hkv) * d].reshape(S, Hkv, d)
    vv = x[:, (Hq + Hkv) * d:].reshape(S, Hkv, d)
    if rope_on:
        qq = om.rope(qq, pos[P:], cfg["rope_theta"])
        kk = om.rope(kk, pos[P:], cfg["rope_theta"])
    if round_qk:
        qq = synth.bf16_round(qq.astype(np.float32)).astype(np.float64)
        kk = synth.bf16_round(kk.astype(np.float32)).astype(np.float64)
    if ents:
        Kp = np.concatenate([entity_kv[(k, i)][0][layer][: used[(k, i)]] for k, i, _ in ents]).astype(np.float64)
        Vp = np.concatenate([entity_kv[(k, i)][1][layer][: used[(k, i)]] for k, i, _ in ents]).astype(np.float64)
        K = np.concatenate([Kp, kk])
        V = np.concatenate([Vp, vv])
    else:
        K, V = kk, vv
    mask = bipartite_mask(seg)[P:, :]
    return om.attention(qq, K, V, mask, Hq // Hkv)

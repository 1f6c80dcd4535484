"""Pins for oracle/model.py.

I4  N = 1: both orderings are an ordinary causal forward -> HuggingFace transformers Qwen2
    in float64 with the same weights (library routine; its RMSNorm, rotary and eager softmax force fp32,
    so those three are patched to fp64 to compare at 1e-10).
I1  cached-prefix reuse == full recompute, UP and IP, incl. ragged items/header.
I2  items are mutually invisible: perturbing item b leaves item a's K/V unchanged; an item's
    standalone KV equals its in-context KV in IP.
I3  candidate permutation equivariance.
I5  UP == IP in the degenerate cases (SURVEY §8(c) issue 1): L=1 without RoPE; |U| = 0.
Guard: a plain causal mask moves z by > 10x the bf16 tolerance, so the
parity tests can see mask bugs.
"""
import numpy as np
import pytest

import synth
from oracle import model as om
from oracle.sequence import build_sequence, bipartite_mask, causal_mask

CFG = synth.model_config("tiny")


def _query(order, n_user=16, n_items=4, item_len=(8, 8), n_instr=2, seed=0, item_ids=None,
           n_header=0, user_id=3):
    ids = item_ids if item_ids is not None else [11, 22, 33, 44][:n_items]
    return synth.make_query(seed, CFG, user_id, n_user, ids, item_len, n_instr, order,
                            n_header=n_header)


@pytest.fixture(scope="module")
def W():
    return synth.Weights(CFG, seed=1)


# ---------------------------------------------------------------------------------- I4
def _hf_forward(cfg, W, tokens):
    import torch
    from transformers import Qwen2Config, Qwen2ForCausalLM
    from transformers.models.qwen2 import modeling_qwen2 as mq

    def rms_fwd(self, x):
        v = x.pow(2).mean(-1, keepdim=True)
        return self.weight * (x * torch.rsqrt(v + self.variance_epsilon))

    def rot_fwd(self, x, position_ids):
        d = cfg["head_dim"]
        inv = 1.0 / (cfg["rope_theta"] ** (torch.arange(0, d, 2, dtype=torch.float64) / d))
        f = position_ids[0].to(torch.float64)[:, None] * inv[None, :]
        emb = torch.cat([f, f], dim=-1)[None]
        return emb.cos().to(x.dtype), emb.sin().to(x.dtype)

    hf_cfg = Qwen2Config(vocab_size=cfg["vocab"], hidden_size=cfg["hidden"],
                         intermediate_size=cfg["ffn"], num_hidden_layers=cfg["layers"],
                         num_attention_heads=cfg["q_heads"], num_key_value_heads=cfg["kv_heads"],
                         head_dim=cfg["head_dim"], max_position_embeddings=4096,
                         rope_theta=cfg["rope_theta"], rms_norm_eps=cfg["rms_eps"],
                         tie_word_embeddings=False, attention_dropout=0.0, use_sliding_window=False)
    hf_cfg._attn_implementation = "eager"
    def eager64(module, query, key, value, attention_mask, scaling, dropout=0.0, **kw):
        ks = mq.repeat_kv(key, module.num_key_value_groups)
        vs = mq.repeat_kv(value, module.num_key_value_groups)
        w = torch.matmul(query, ks.transpose(2, 3)) * scaling
        if attention_mask is not None:
            w = w + attention_mask
        w = torch.softmax(w, dim=-1)            # upstream forces fp32 here
        return torch.matmul(w, vs).transpose(1, 2).contiguous(), w

    old = (mq.Qwen2RMSNorm.forward, mq.Qwen2RotaryEmbedding.forward, mq.eager_attention_forward)
    mq.Qwen2RMSNorm.forward, mq.Qwen2RotaryEmbedding.forward = rms_fwd, rot_fwd
    mq.eager_attention_forward = eager64
    try:
        m = Qwen2ForCausalLM(hf_cfg).to(torch.float64).eval()
        H, d, Hq, Hkv, F = cfg["hidden"], cfg["head_dim"], cfg["q_heads"], cfg["kv_heads"], cfg["ffn"]
        t = lambda a: torch.tensor(np.asarray(a, dtype=np.float64))
        with torch.no_grad():
            m.model.embed_tokens.weight.copy_(t(W.embed_full()))
            for l, layer in enumerate(m.model.layers):
                w = W.layer(l)
                a = layer.self_attn
                a.q_proj.weight.copy_(t(w["wqkv"][: Hq * d])); a.q_proj.bias.copy_(t(w["bqkv"][: Hq * d]))
                a.k_proj.weight.copy_(t(w["wqkv"][Hq * d:(Hq + Hkv) * d])); a.k_proj.bias.copy_(t(w["bqkv"][Hq * d:(Hq + Hkv) * d]))
                a.v_proj.weight.copy_(t(w["wqkv"][(Hq + Hkv) * d:])); a.v_proj.bias.copy_(t(w["bqkv"][(Hq + Hkv) * d:]))
                a.o_proj.weight.copy_(t(w["wo"]))
                layer.input_layernorm.weight.copy_(t(w["ln1"]))
                layer.post_attention_layernorm.weight.copy_(t(w["ln2"]))
                layer.mlp.gate_proj.weight.copy_(t(w["wgu"][:F]))
                layer.mlp.up_proj.weight.copy_(t(w["wgu"][F:]))
                layer.mlp.down_proj.weight.copy_(t(w["wd"]))
            m.model.norm.weight.copy_(t(W.final_norm()))
            ids = torch.tensor(np.asarray(tokens, dtype=np.int64))[None]
            out = m.model(input_ids=ids, position_ids=torch.arange(len(tokens))[None])
            return out.last_hidden_state[0].numpy()
    finally:
        mq.Qwen2RMSNorm.forward, mq.Qwen2RotaryEmbedding.forward, mq.eager_attention_forward = old


@pytest.mark.parametrize("order", ["UP", "IP"])
def test_I4_single_item_is_plain_causal_forward_vs_transformers(W, order):
    q = _query(order, n_items=1, item_len=(5, 5))
    tokens, seg, pos = build_sequence(order, q.user_tok, q.item_toks, q.instr_tok)
    assert np.array_equal(pos, np.arange(len(tokens)))          # N=1: ordinary positions
    assert np.array_equal(bipartite_mask(seg), causal_mask(len(tokens)))
    h, _ = om.forward_full(CFG, W, tokens, pos, bipartite_mask(seg))
    ref_final = _hf_forward(CFG, W, tokens)                      # HF applies the final norm
    ours_final = om.rmsnorm(h, np.asarray(W.final_norm(), np.float64), CFG["rms_eps"])
    np.testing.assert_allclose(ours_final, ref_final, rtol=1e-10, atol=1e-10)


# ---------------------------------------------------------------------------------- I1
@pytest.mark.parametrize("order", ["UP", "IP"])
@pytest.mark.parametrize("item_len,n_header", [((8, 8), 0), ((12, 20), 0), ((3, 9), 2)])
def test_I1_cached_equals_recompute(W, order, item_len, n_header):
    if order == "UP" and n_header:
        pytest.skip("header is IP-only")
    q = _query(order, item_len=item_len, n_header=n_header)
    full = om.run_query(CFG, W, q, "full")
    cached = om.run_query(CFG, W, q, "cached")
    np.testing.assert_allclose(cached["hf"], full["hf"], rtol=1e-11, atol=1e-11)
    np.testing.assert_allclose(cached["z"], full["z"], rtol=1e-11, atol=1e-11)


# ---------------------------------------------------------------------------------- I2
@pytest.mark.parametrize("order", ["UP", "IP"])
def test_I2_items_mutually_invisible(W, order):
    q = _query(order)
    toks, seg, pos = build_sequence(order, q.user_tok, q.item_toks, q.instr_tok)
    _, kv1 = om.forward_full(CFG, W, toks, pos, bipartite_mask(seg), keep_kv=True)
    toks2 = toks.copy()
    toks2[seg == 2] = (toks2[seg == 2] + 7) % CFG["vocab"]   # perturb item b = 2
    _, kv2 = om.forward_full(CFG, W, toks2, pos, bipartite_mask(seg), keep_kv=True)
    for a in (0, 1, 3):
        sel = seg == a
        for l in range(CFG["layers"]):
            assert np.array_equal(kv1[l][0][sel], kv2[l][0][sel])
            assert np.array_equal(kv1[l][1][sel], kv2[l][1][sel])
    assert not np.allclose(kv1[0][0][seg == 2], kv2[0][0][seg == 2])


def test_I2_item_standalone_kv_equals_in_context_kv(W):
    q = _query("IP", item_len=(5, 11))
    toks, seg, pos = build_sequence("IP", q.user_tok, q.item_toks, q.instr_tok)
    _, kv = om.forward_full(CFG, W, toks, pos, bipartite_mask(seg), keep_kv=True)
    for i, t in enumerate(q.item_toks):
        alone = om.entity_kv(CFG, W, t, 0)
        for l in range(CFG["layers"]):
            np.testing.assert_allclose(alone[l][0], kv[l][0][seg == i], rtol=1e-12, atol=1e-12)
            np.testing.assert_allclose(alone[l][1], kv[l][1][seg == i], rtol=1e-12, atol=1e-12)


# ---------------------------------------------------------------------------------- I3
@pytest.mark.parametrize("order", ["UP", "IP"])
def test_I3_permutation_equivariance(W, order):
    ids = [11, 22, 33, 44]
    perm = [2, 0, 3, 1]
    a = om.run_query(CFG, W, _query(order, item_ids=ids, item_len=(4, 9)), "full")
    b = om.run_query(CFG, W, _query(order, item_ids=[ids[p] for p in perm], item_len=(4, 9)), "full")
    np.testing.assert_allclose(b["s"], a["s"][perm], rtol=1e-11, atol=1e-12)
    np.testing.assert_allclose(b["z"], a["z"][perm], rtol=1e-11, atol=1e-12)


# ---------------------------------------------------------------------------------- I5
def test_I5_up_equals_ip_single_layer_without_rope():
    cfg = dict(CFG, layers=1)
    W1 = synth.Weights(cfg, seed=5)
    res = {}
    for order in ("UP", "IP"):
        q = synth.make_query(0, cfg, 3, 16, [11, 22, 33, 44], (8, 8), 2, order)
        res[order] = om.run_query(cfg, W1, q, "full", rope_on=False)
    np.testing.assert_allclose(res["UP"]["s"], res["IP"]["s"], rtol=1e-11, atol=1e-13)


def test_I5_up_equals_ip_without_user_tokens(W):
    res = {o: om.run_query(CFG, W, _query(o, n_user=0), "full") for o in ("UP", "IP")}
    np.testing.assert_array_equal(res["UP"]["z"], res["IP"]["z"])


def test_up_vs_ip_general_case_is_reported_not_asserted(W):
    """Parity unpinned (SURVEY §8(c) issue 1): UP and IP attend different key sets."""
    res = {o: om.run_query(CFG, W, _query(o), "full") for o in ("UP", "IP")}
    diff = float(np.max(np.abs(res["UP"]["s"] - res["IP"]["s"])))
    print(f"max|s_UP - s_IP| = {diff:.4g}")
    assert np.isfinite(diff)


# ------------------------------------------------------------------------------ guard
@pytest.mark.parametrize("order", ["UP", "IP"])
def test_mask_sensitivity_guard(W, order):
    q = _query(order)
    good = om.run_query(CFG, W, q, "full")
    bad = om.run_query(CFG, W, q, "full", mask_fn=lambda seg: causal_mask(len(seg)))
    assert np.max(np.abs(good["z"] - bad["z"])) > 10 * 2e-2


@pytest.mark.parametrize("order", ["UP", "IP"])
def test_mask_sensitivity_guard_small_gqa6(order):
    """Same guard at the Qwen-like "small" GPU-parity config (g = 6, d = 128, init 0.02)."""
    cfg = synth.model_config("small")
    Ws = synth.Weights(cfg, seed=1)
    q = synth.make_query(3, cfg, 6, 100, list(range(200, 220)), (16, 16), 8, order)
    good = om.run_query(cfg, Ws, q, "full")
    bad = om.run_query(cfg, Ws, q, "full", mask_fn=lambda seg: causal_mask(len(seg)))
    assert np.max(np.abs(good["z"] - bad["z"])) > 10 * 2e-2


# ------------------------------------------------------------------------- attention
def test_attention_dense_block_is_textbook_softmax():
    from scipy.special import softmax
    rng = np.random.default_rng(0)
    T, Tk, Hq, Hkv, d = 5, 7, 4, 2, 8
    q, k, v = rng.normal(size=(T, Hq, d)), rng.normal(size=(Tk, Hkv, d)), rng.normal(size=(Tk, Hkv, d))
    o = om.attention(q, k, v, np.ones((T, Tk), bool), Hq // Hkv)
    for j in range(Hq):
        ref = softmax(q[:, j] @ k[:, j // 2].T / np.sqrt(d), axis=1) @ v[:, j // 2]
        np.testing.assert_allclose(o[:, j], ref, rtol=1e-12, atol=1e-12)


def test_attention_single_visible_key_returns_its_value():
    rng = np.random.default_rng(1)
    q, k, v = rng.normal(size=(3, 2, 4)), rng.normal(size=(3, 1, 4)), rng.normal(size=(3, 1, 4))
    mask = np.eye(3, dtype=bool)
    o = om.attention(q, k, v, mask, 2)
    for t in range(3):
        np.testing.assert_allclose(o[t, 0], v[t, 0], rtol=0, atol=1e-15)
        np.testing.assert_allclose(o[t, 1], v[t, 0], rtol=0, atol=1e-15)


def test_rope_rotation_properties():
    rng = np.random.default_rng(2)
    x = rng.normal(size=(6, 3, 8))
    pos = np.arange(6)
    r = om.rope(x, pos, 10000.0)
    # a rotation preserves norms of every (i, i + d/2) pair; position 0 is the identity
    np.testing.assert_allclose(np.linalg.norm(r, axis=-1), np.linalg.norm(x, axis=-1), rtol=1e-12)
    np.testing.assert_allclose(r[0], x[0], rtol=0, atol=0)
    # relative-position property: <R(p)a, R(p')b> depends only on p - p'
    a, b = rng.normal(size=(1, 1, 8)), rng.normal(size=(1, 1, 8))
    dot = lambda p1, p2: float(np.sum(om.rope(a, np.array([p1]), 1e4) * om.rope(b, np.array([p2]), 1e4)))
    assert abs(dot(5, 2) - dot(13, 10)) < 1e-12


@pytest.mark.parametrize("order", ["UP", "IP"])
def test_mask_sensitivity_guard_small64(order):
    """Guard at the head_dim-64 GQA-4 parity config (Llama3-1B's head shape, Table 2)."""
    cfg = synth.model_config("small64")
    Ws = synth.Weights(cfg, seed=1)
    q = synth.make_query(8, cfg, 9, 120, list(range(400, 424)), (16, 16), 8, order)
    good = om.run_query(cfg, Ws, q, "full")
    bad = om.run_query(cfg, Ws, q, "full", mask_fn=lambda seg: causal_mask(len(seg)))
    assert np.max(np.abs(good["z"] - bad["z"])) > 10 * 2e-2


# ---------------------------------------------- multi-discriminant variant (R20)
def _mq(seed=0, items=(11, 22, 33, 44), n_user=16):
    q = synth.make_query(seed, CFG, 3, n_user, list(items), (8, 8), 2, "UP")
    q.multi_disc = True
    return q


def test_multi_disc_cached_equals_full(W):
    """I1 for the per-item discriminants: serving U from its cached KV changes nothing."""
    q = _mq()
    a = om.run_query_multi(CFG, W, q, "full")
    b = om.run_query_multi(CFG, W, q, "cached")
    np.testing.assert_allclose(a["hf"], b["hf"], rtol=1e-10, atol=1e-10)
    np.testing.assert_allclose(a["s"], b["s"], rtol=1e-10, atol=1e-12)


def test_multi_disc_item_independence(W):
    """I2: item i's discriminant sees U and its own item only — changing another item's
    tokens leaves hf_i (and z_i) unchanged, while hf_j of the changed item moves."""
    q = _mq()
    a = om.run_query_multi(CFG, W, q, "full")
    q2 = _mq()
    q2.item_toks = list(q2.item_toks)
    q2.item_toks[2] = (np.asarray(q2.item_toks[2]) + 7) % CFG["vocab"]
    b = om.run_query_multi(CFG, W, q2, "full")
    for i in (0, 1, 3):
        np.testing.assert_allclose(a["hf"][i], b["hf"][i], rtol=1e-12, atol=1e-12)
    assert np.max(np.abs(a["hf"][2] - b["hf"][2])) > 1e-3


def test_multi_disc_permutation_equivariance(W):
    """I3: permuting the candidates permutes the scores."""
    a = om.run_query_multi(CFG, W, _mq(items=(11, 22, 33, 44)), "full")
    b = om.run_query_multi(CFG, W, _mq(items=(33, 11, 44, 22)), "full")
    np.testing.assert_allclose(b["s"], a["s"][[2, 0, 3, 1]], rtol=1e-10, atol=1e-12)


def test_multi_disc_rows_are_plain_causal_forwards_vs_transformers(W):
    """Pins WHICH row is item i's discriminant and what it sees (R20): in
    User-as-prefix order item i's tokens attend to U and to their own item only, at positions
    |U| + j — exactly an ordinary causal forward of the sequence [U, I_i] — so its discriminant
    (item i's LAST token) must equal HuggingFace Qwen2's final-normed last hidden state of [U, I_i],
    and z_i = W_out[v_i] . that state.  Ragged items: the first token, an off-by-one inside the item
    or another item's row would each fail."""
    q = synth.make_query(2, CFG, 9, 11, [5, 6, 7], (3, 9), 2, "UP")
    assert len({len(t) for t in q.item_toks}) > 1
    q.multi_disc = True
    a = om.run_query_multi(CFG, W, q, "full")
    for i, t in enumerate(q.item_toks):
        ref = _hf_forward(CFG, W, np.concatenate([q.user_tok, t]))[-1]
        np.testing.assert_allclose(a["hf"][i], ref, rtol=1e-10, atol=1e-10)
        zi = float(np.asarray(W.lm_head_rows([q.labels[i]]), np.float64)[0] @ ref)
        np.testing.assert_allclose(a["z"][i], zi, rtol=1e-10, atol=1e-10)

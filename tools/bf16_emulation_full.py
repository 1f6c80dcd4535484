"""Full-size (Qwen2-1.5B, 28 layers) emulation of the GPU's bf16 rounding points next to the fp64
oracle, layer by layer, on one configs[1] IP request (full recompute of the same prompt): shows
how much of the GPU-vs-oracle difference an ideal bf16 pipeline already has (R12).
usage: python tools/bf16_emulation_full.py [mlp_std] [attn_std] [layers] [model] [n_user] [n_items] [seed]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, synth
from oracle import model as om
from oracle.sequence import build_sequence, bipartite_mask
bf = lambda a: synth.bf16_round(np.asarray(a, np.float32)).astype(np.float64)
cfg = synth.model_config(sys.argv[4] if len(sys.argv) > 4 else "qwen2-1.5b")
if len(sys.argv) > 3: cfg["layers"] = int(sys.argv[3])
if len(sys.argv) > 1: cfg["mlp_std"] = float(sys.argv[1])
W = synth.Weights(cfg, seed=int(sys.argv[7]) if len(sys.argv) > 7 else 1, std=float(sys.argv[2]) if len(sys.argv) > 2 else None)
if len(sys.argv) > 2: W.mlp_std = float(sys.argv[1])
n_user = int(sys.argv[5]) if len(sys.argv) > 5 else 512
n_items = int(sys.argv[6]) if len(sys.argv) > 6 else 100
H, d, Hq, Hkv, F = cfg["hidden"], cfg["head_dim"], cfg["q_heads"], cfg["kv_heads"], cfg["ffn"]
rng = np.random.default_rng(7)
q = synth.make_query(0, cfg, 1000, n_user, synth.distinct_label_items(0, cfg, n_items, rng, 8192, synth.zipf_weights(8192)), (16, 16), 8, "IP")
toks, seg, pos = build_sequence(q.order, q.user_tok, q.item_toks, q.instr_tok)
mask = bipartite_mask(seg)
h64 = np.asarray(W.embed_rows(toks), np.float64)
h16 = h64.copy()
def layer_bf16(w, h, S):
    a = bf(om.rmsnorm(h, w["ln1"], 1e-6))
    qkv = bf(a @ np.asarray(w["wqkv"], np.float64).T + w["bqkv"])
    qq = qkv[:, :Hq*d].reshape(S, Hq, d); kk = qkv[:, Hq*d:(Hq+Hkv)*d].reshape(S, Hkv, d); vv = qkv[:, (Hq+Hkv)*d:].reshape(S, Hkv, d)
    qq = bf(om.rope(qq, pos, cfg["rope_theta"])); kk = bf(om.rope(kk, pos, cfg["rope_theta"]))
    o = np.zeros((S, Hq, d))
    for j in range(Hq):
        s = qq[:, j] @ kk[:, j // (Hq // Hkv)].T / np.sqrt(d); s = np.where(mask, s, -np.inf)
        m = s.max(1, keepdims=True); p = np.where(mask, np.exp(s - m), 0)
        o[:, j] = (bf(p) @ vv[:, j // (Hq // Hkv)]) / p.sum(1, keepdims=True)
    o = bf(o)
    h = h + o.reshape(S, -1) @ np.asarray(w["wo"], np.float64).T
    b = bf(om.rmsnorm(h, w["ln2"], 1e-6))
    gu = bf(b @ np.asarray(w["wgu"], np.float64).T)  # (GPU: SwiGLU from fp32 accumulators; bf16 here is pessimistic)
    act = bf(om.silu(gu[:, :F]) * gu[:, F:])
    return h + act @ np.asarray(w["wd"], np.float64).T
fn = np.asarray(W.final_norm(), np.float64)
for l in range(cfg["layers"]):
    t0 = time.time()
    w = W.layer(l)
    h64, _, _ = om.layer_forward(cfg, w, h64, pos, None, None, mask)
    h16 = layer_bf16(w, h16, len(toks))
    rel = np.linalg.norm(h16[-1] - h64[-1]) / np.linalg.norm(h64[-1])
    hf64 = om.rmsnorm(h64[-1], fn, 1e-6); hf16 = om.rmsnorm(h16[-1], fn, 1e-6)
    exc = np.max(np.abs(hf16 - hf64) - (0.02 + 0.02 * np.abs(hf64)))
    print(f"layer {l:2d} rms(h_last) {np.sqrt(np.mean(h64[-1]**2)):.4f} rel err {rel:.2e} hf max|err| {np.abs(hf16-hf64).max():.4f} excess {exc:+.4f}  ({time.time()-t0:.1f}s)", flush=True)

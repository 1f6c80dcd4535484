"""Seeded synthetic inputs shared by the oracle tests, the CUDA-path tests and bench.py.

This module holds NO arithmetic of the method (no attention, no masks, no positions,
no model math).  It only draws random numbers and shapes them into model weights,
token ids and query descriptions, so that both sides of every parity test (``oracle/``
and the CUDA path under ``paper_conf_asplos_0017wzlxszh0w26_b200/``) see identical
inputs.  The recipe is stated in DESIGN.md §"Input recipe" and follows SURVEY.md §8(d):

* weights N(0, 0.02) for every matrix and bias of the Qwen-width models (the token
  embedding included: an N(0,1) embedding hides mask bugs, SURVEY §8(c) issue 11b) and
  for the narrow tiny config (H=64) N(0, 1/H) for the embedding and attention matrices and
  N(0, 0.05^2) for the MLP matrices; RMSNorm gains 1 + N(0, 0.1);
  every value rounded to bf16 (RNE) so that both sides use exactly the same numbers;
* token ids uniform in [0, vocab); item tokens and identifier labels are a function of
  the item id (the same item has the same tokens in every query, which is what makes its
  KV cache reusable), user tokens a function of the user id;
* item hotness Zipf(s) over the corpus (~90% of accesses on the top 10% of items);
  user lengths lognormal(median 1500, sigma 0.8) clipped to [64, 8192] (Table 1).

Every generator is counter-based: a tensor block is drawn from
``np.random.default_rng(SeedSequence([seed, tag, layer, block]))`` so any slice of a
large tensor (e.g. 1024 rows of a 151936-row embedding) can be regenerated on its own.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Dict, List, Optional, Sequence

import numpy as np

# --------------------------------------------------------------------------------------
# model shapes (SURVEY.md §8 "Model shapes"; tiny = BASELINE.json configs[0])
# --------------------------------------------------------------------------------------

MODEL_CONFIGS: Dict[str, dict] = {
    # configs[0]: 2 layers, hidden 64, 4 heads (2 KV); d=16, F=256, vocab=512 proposed
    "tiny": dict(layers=2, hidden=64, q_heads=4, kv_heads=2, head_dim=16, ffn=256,
                 vocab=512, rope_theta=10000.0, rms_eps=1e-6, tied=False, mlp_std=0.05),
    # a Qwen-like (g=6, d=128) small model used for multi-tile GPU parity at oracle speed
    "small": dict(layers=2, hidden=768, q_heads=6, kv_heads=1, head_dim=128, ffn=1024,
                  vocab=4096, rope_theta=1e6, rms_eps=1e-6, tied=False, mlp_std=0.01),
    # the same at GQA group 7 (Qwen2-7B's 28 Q / 4 KV heads: 18 tokens x 7 heads per q-tile)
    "small7": dict(layers=2, hidden=896, q_heads=7, kv_heads=1, head_dim=128, ffn=1024,
                   vocab=4096, rope_theta=1e6, rms_eps=1e-6, tied=False, mlp_std=0.01),
    # the head_dim-64 GQA-4 shape of Llama3-1B (Table 2: 8 KV heads, d = 64) at parity size
    "small64": dict(layers=2, hidden=512, q_heads=8, kv_heads=2, head_dim=64, ffn=1024,
                    vocab=4096, rope_theta=5e5, rms_eps=1e-5, tied=False, mlp_std=0.01),
    # Llama3-1B shape (Table 2: 16 layers, 8 KV heads, d 64; hidden / F / vocab /
    # theta / eps / tying from the public Llama-3.2-1B config; weights random, shapes only; the
    # Qwen2-style qkv bias is kept (drawn, not zero) since the shapes are what matter)
    "llama3-1b": dict(layers=16, hidden=2048, q_heads=32, kv_heads=8, head_dim=64, ffn=8192,
                      vocab=128256, rope_theta=5e5, rms_eps=1e-5, tied=True),
    # Qwen2-1.5B shape (Table 2 P:396-403 + public config for F / vocab / theta / eps)
    "qwen2-1.5b": dict(layers=28, hidden=1536, q_heads=12, kv_heads=2, head_dim=128,
                       ffn=8960, vocab=151936, rope_theta=1e6, rms_eps=1e-6, tied=True),
    # Qwen2-7B shape
    "qwen2-7b": dict(layers=28, hidden=3584, q_heads=28, kv_heads=4, head_dim=128,
                     ffn=18944, vocab=152064, rope_theta=1e6, rms_eps=1e-6, tied=False),
}

_TAG = dict(embed=1, lm_head=2, final_norm=3, ln1=10, wqkv=11, bqkv=12, wo=13, ln2=14,
            wgu=15, wd=16, user_tok=40, item_tok=41, item_label=42, instr_tok=43,
            header_tok=44, user_len=45, query=46, kv=47, trace=48)

ROW_BLOCK = 1024


def model_config(name: str) -> dict:
    return dict(MODEL_CONFIGS[name])


def bf16_round(x: np.ndarray) -> np.ndarray:
    """Round float32 values to the nearest bf16 (round-to-nearest-even); returns float32."""
    x = np.ascontiguousarray(x, dtype=np.float32)
    u = x.view(np.uint32).astype(np.uint64)
    lsb = (u >> 16) & 1
    u = (u + 0x7FFF + lsb) & 0xFFFF0000
    return u.astype(np.uint32).view(np.float32).reshape(x.shape)


def _rng(*key: int) -> np.random.Generator:
    return np.random.default_rng(np.random.SeedSequence([int(k) & 0xFFFFFFFF for k in key]))


def gen_rows(seed: int, tag: int, layer: int, n_rows: int, n_cols: int, std: float,
             mean: float = 0.0, row0: int = 0, row1: Optional[int] = None) -> np.ndarray:
    """Rows [row0,row1) of an n_rows x n_cols tensor ~ N(mean, std^2), bf16-rounded."""
    row1 = n_rows if row1 is None else row1
    assert 0 <= row0 <= row1 <= n_rows
    out = np.empty((row1 - row0, n_cols), dtype=np.float32)
    b0, b1 = row0 // ROW_BLOCK, (row1 + ROW_BLOCK - 1) // ROW_BLOCK
    for b in range(b0, b1):
        r_lo, r_hi = b * ROW_BLOCK, min(n_rows, (b + 1) * ROW_BLOCK)
        blk = _rng(seed, tag, layer, b).standard_normal((r_hi - r_lo, n_cols), dtype=np.float32)
        blk = blk * np.float32(std) + np.float32(mean)
        s_lo, s_hi = max(r_lo, row0), min(r_hi, row1)
        out[s_lo - row0:s_hi - row0] = blk[s_lo - r_lo:s_hi - r_lo]
    return bf16_round(out)


def gen_rows_at(seed: int, tag: int, layer: int, n_rows: int, n_cols: int, std: float,
                rows: Sequence[int], mean: float = 0.0) -> np.ndarray:
    """Selected rows (any order) of the tensor gen_rows would produce."""
    rows = np.asarray(rows, dtype=np.int64)
    out = np.empty((len(rows), n_cols), dtype=np.float32)
    blocks = np.unique(rows // ROW_BLOCK)
    for b in blocks:
        r_lo = int(b) * ROW_BLOCK
        blk = gen_rows(seed, tag, layer, n_rows, n_cols, std, mean, r_lo,
                       min(n_rows, r_lo + ROW_BLOCK))
        sel = np.nonzero(rows // ROW_BLOCK == b)[0]
        out[sel] = blk[rows[sel] - r_lo]
    return out


class Weights:
    """Random-init weights of a Qwen2-shaped model (no trained weights exist).

    Layout (the C ABI's, include/bat.h): embed [vocab][H]; lm_head [vocab][H] (== embed
    when tied); final_norm [H]; per layer: ln1 [H], wqkv [(Hq+2Hkv)d][H] (q rows, then k,
    then v), bqkv [(Hq+2Hkv)d], wo [H][Hq d], ln2 [H], wgu [2F][H] (gate rows then up rows),
    wd [H][F].  All float32 arrays holding bf16-exact values.
    """

    def __init__(self, cfg: dict, seed: int = 0, std: Optional[float] = None):
        self.cfg = dict(cfg)
        self.seed = int(seed)
        H, V = cfg["hidden"], cfg["vocab"]
        # 0.02 (HF initializer_range) for the Qwen-width models; fan-in 1/sqrt(H) for the
        # tiny config, where 0.02 leaves attention so flat that a wrong mask moves the
        # logits by less than 10x the bf16 tolerance (tests/test_oracle_model.py guard)
        self.std = float(std) if std is not None else (0.02 if H >= 512 else 1.0 / np.sqrt(H))
        # parity configs: smaller MLP matrices (tiny N(0, 0.05^2), small N(0, 0.01^2)) — with
        # larger MLP weights the 2-layer nets amplify bf16 rounding up to ~1x the 2e-2 tolerance
        # on hf even in an ideal bf16 pipeline (tools/bf16_emulation.py; R12)
        self.mlp_std = float(cfg.get("mlp_std", self.std)) if std is None else self.std
        # tiny (H=64): a tied 0.02 head gives logit std ~0.16; use N(0, 1/sqrt(H)) untied
        self.lm_std = (1.0 / np.sqrt(H)) if H < 512 else self.std
        self._cache: Dict[int, dict] = {}

    # -- global tensors ------------------------------------------------------------
    def embed_rows(self, rows) -> np.ndarray:
        c = self.cfg
        return gen_rows_at(self.seed, _TAG["embed"], 0, c["vocab"], c["hidden"], self.std, rows)

    def embed_full(self) -> np.ndarray:
        c = self.cfg
        return gen_rows(self.seed, _TAG["embed"], 0, c["vocab"], c["hidden"], self.std)

    def lm_head_rows(self, rows) -> np.ndarray:
        if self.cfg["tied"]:
            return self.embed_rows(rows)
        c = self.cfg
        return gen_rows_at(self.seed, _TAG["lm_head"], 0, c["vocab"], c["hidden"], self.lm_std, rows)

    def lm_head_full(self) -> np.ndarray:
        if self.cfg["tied"]:
            return self.embed_full()
        c = self.cfg
        return gen_rows(self.seed, _TAG["lm_head"], 0, c["vocab"], c["hidden"], self.lm_std)

    def final_norm(self) -> np.ndarray:
        return gen_rows(self.seed, _TAG["final_norm"], 0, 1, self.cfg["hidden"], 0.1, 1.0)[0]

    # -- per-layer tensors -----------------------------------------------------------
    def layer(self, l: int) -> dict:
        if l in self._cache:
            return self._cache[l]
        c, s, sd = self.cfg, self.seed, self.std
        H, d, Hq, Hkv, F = c["hidden"], c["head_dim"], c["q_heads"], c["kv_heads"], c["ffn"]
        nqkv = (Hq + 2 * Hkv) * d
        w = dict(
            ln1=gen_rows(s, _TAG["ln1"], l, 1, H, 0.1, 1.0)[0],
            wqkv=gen_rows(s, _TAG["wqkv"], l, nqkv, H, sd),
            bqkv=gen_rows(s, _TAG["bqkv"], l, 1, nqkv, sd)[0],
            wo=gen_rows(s, _TAG["wo"], l, H, Hq * d, sd),
            ln2=gen_rows(s, _TAG["ln2"], l, 1, H, 0.1, 1.0)[0],
            wgu=gen_rows(s, _TAG["wgu"], l, 2 * F, H, self.mlp_std),
            wd=gen_rows(s, _TAG["wd"], l, H, F, self.mlp_std),
        )
        if c["layers"] * H <= 4096:  # small models: keep in memory
            self._cache[l] = w
        return w

    LAYER_KEYS = ("ln1", "wqkv", "bqkv", "wo", "ln2", "wgu", "wd")


# --------------------------------------------------------------------------------------
# tokens of users / items / instructions (functions of the entity id)
# --------------------------------------------------------------------------------------

def user_tokens(seed: int, user_id: int, n: int, vocab: int) -> np.ndarray:
    return _rng(seed, _TAG["user_tok"], user_id).integers(0, vocab, size=n, dtype=np.int64).astype(np.int32)


def item_tokens(seed: int, item_id: int, n: int, vocab: int) -> np.ndarray:
    return _rng(seed, _TAG["item_tok"], item_id).integers(0, vocab, size=n, dtype=np.int64).astype(np.int32)


def item_label(seed: int, item_id: int, vocab: int) -> int:
    """Identifier token v_i of item i, intrinsic to the item."""
    return int(_rng(seed, _TAG["item_label"], item_id).integers(0, vocab))


def instr_tokens(seed: int, n: int, vocab: int) -> np.ndarray:
    return _rng(seed, _TAG["instr_tok"], 0).integers(0, vocab, size=n, dtype=np.int64).astype(np.int32)


def header_tokens(seed: int, n: int, vocab: int) -> np.ndarray:
    return _rng(seed, _TAG["header_tok"], 0).integers(0, vocab, size=n, dtype=np.int64).astype(np.int32)


def item_length(item_id: int, lo: int, hi: int, seed: int = 0) -> int:
    """Per-item token count in [lo, hi] (fixed when lo == hi)."""
    if lo == hi:
        return lo
    return int(_rng(seed, _TAG["item_tok"], item_id, 7).integers(lo, hi + 1))


@dataclass
class Query:
    """One ranking request: a user, N candidate items, instruction tokens.

    ``order`` is the prefix side chosen for this request ("UP" P:249 or "IP" P:253);
    ``use_cache`` False means full recompute (RE) of the same ordered sequence.
    """
    user_id: int
    user_tok: np.ndarray
    item_ids: np.ndarray
    item_toks: List[np.ndarray]
    labels: np.ndarray
    instr_tok: np.ndarray
    order: str = "IP"
    use_cache: bool = True
    header_id: int = -1
    header_tok: np.ndarray = field(default_factory=lambda: np.zeros(0, np.int32))
    multi_disc: bool = False  # one discriminant token per item (UP only)
    pic_tail: int = 0         # IP selective recompute: last k tokens of every item (reading R25)

    @property
    def n_items(self) -> int:
        return len(self.item_ids)


def make_query(seed: int, cfg: dict, user_id: int, n_user: int, item_ids: Sequence[int],
               item_len=(16, 16), n_instr: int = 8, order: str = "IP",
               use_cache: bool = True, n_header: int = 0) -> Query:
    V = cfg["vocab"]
    item_ids = np.asarray(item_ids, dtype=np.int64)
    lo, hi = item_len
    toks = [item_tokens(seed, int(i), item_length(int(i), lo, hi, seed), V) for i in item_ids]
    labels = np.array([item_label(seed, int(i), V) for i in item_ids], dtype=np.int32)
    return Query(user_id=int(user_id), user_tok=user_tokens(seed, user_id, n_user, V),
                 item_ids=item_ids, item_toks=toks, labels=labels,
                 instr_tok=instr_tokens(seed, n_instr, V), order=order, use_cache=use_cache,
                 header_id=(0 if n_header else -1), header_tok=header_tokens(seed, n_header, V))


def distinct_label_items(seed: int, cfg: dict, n_items: int, rng: np.random.Generator,
                         corpus: int, weights: Optional[np.ndarray] = None) -> np.ndarray:
    """Sample n distinct candidate item ids whose labels v_i are distinct."""
    V = cfg["vocab"]
    chosen: List[int] = []
    seen_items, seen_labels = set(), set()
    while len(chosen) < n_items:
        if weights is None:
            draw = rng.integers(0, corpus, size=2 * n_items)
        else:
            draw = rng.choice(corpus, size=2 * n_items, p=weights)
        for i in draw:
            i = int(i)
            if len(chosen) == n_items:
                break
            if i in seen_items:
                continue
            lab = item_label(seed, i, V)
            if lab in seen_labels:
                continue
            seen_items.add(i)
            seen_labels.add(lab)
            chosen.append(i)
    return np.array(chosen, dtype=np.int64)


def zipf_weights(n: int, s: float = 1.093) -> np.ndarray:
    """Item access probabilities ~ rank^-s; s=1.093 puts ~90% of mass on the top 10% of
    a 262,144-item corpus (solved in SURVEY §8(d))."""
    w = np.arange(1, n + 1, dtype=np.float64) ** (-s)
    return w / w.sum()


def user_lengths(seed: int, n: int, median: float = 1500.0, sigma: float = 0.8,
                 lo: int = 64, hi: int = 8192) -> np.ndarray:
    r = _rng(seed, _TAG["user_len"])
    x = np.exp(np.log(median) + sigma * r.standard_normal(n))
    return np.clip(np.round(x), lo, hi).astype(np.int64)


def random_kv(seed: int, entity_key: int, layers: int, n: int, kv_heads: int, head_dim: int,
              std: float = 1.0) -> np.ndarray:
    """Random bf16 K/V [layers][2][n][Hkv][d] for corpus-scale throughput runs, where only
    timing matters (SURVEY §8(d) "Prefix KV")."""
    r = _rng(seed, _TAG["kv"], entity_key)
    x = r.standard_normal((layers, 2, n, kv_heads, head_dim), dtype=np.float32) * np.float32(std)
    return bf16_round(x)


def request_trace(seed: int, n_requests: int, n_users: int, activity_s: float = 1.2,
                  rate: float = 50.0, tau_i: int = 1600, median: float = 1500.0,
                  sigma: float = 0.8):
    """Synthetic ranking-request trace for the prompt scheduler (the real
    traces are out of scope): user activity Zipf(activity_s) over n_users (a long tail of
    inactive users, P:284 / Fig. 2(c)), user profile lengths lognormal (Table 1),
    Poisson arrivals at `rate` requests per time unit, tau_i item tokens per request
    (100 candidates x 16 tokens).  Returns [(time, user_id, tau_u, tau_i)], times increasing."""
    r = _rng(seed, _TAG["trace"])
    p = np.arange(1, n_users + 1, dtype=np.float64) ** (-activity_s)
    p /= p.sum()
    users = r.choice(n_users, size=n_requests, p=p)
    lens = user_lengths(seed, n_users, median=median, sigma=sigma)
    times = np.cumsum(r.exponential(1.0 / rate, size=n_requests))
    return [(float(t), int(u), int(lens[u]), int(tau_i)) for t, u in zip(times, users)]

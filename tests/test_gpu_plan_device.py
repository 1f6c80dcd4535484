"""Bit-exact check of the indexing the attention kernel actually consumes (north_star: "page-table
and indexing results must match bit-exact"), against the oracle's brute-force pair enumeration
(oracle/plan.py, SURVEY §8(c) "Plan definition").

bat_plan_build uploads the host plan and computes the partial-tile visibility masks ON THE
DEVICE (mask_kernel); bat_plan_export_device reads that device image back and decodes it the way
attn_tc_kernel reads it: the work list of every KV head (q-tile pairs, listed k-tiles, per-q-tile
state 0/1/2), the page ids the loader copies per k-tile, and the mask bits of partial tiles.
Asserted for every request of the batch:
  * VIS (layers 1..L-1): the decoded (row, key slot) visibility == the oracle's explicit
    visibility over every pair (dead tiles unlisted, full tiles all-visible, partial = mask bits);
  * VIS_LAST (last layer, P:173 trim): the same for the rows of the last q-tile, nothing else;
  * KPAGES: a k-tile is loaded iff some q-tile of the request has a visible pair in it (exact
    block-skip), with the oracle's page ids (prefix pages from the pool index, suffix scratch
    pages, the all-zero page as 8-page padding);
  * every KV head sees the same lists (checked inside the export: BAT_E_STATE otherwise);
  * STAGE: the destinations the fused QKV epilogue (a4) derives for every suffix row from the
    device row map — global q-tile, suffix page, slot — equal the oracle's.
Batches: configs[1] exactly as bench.py builds it (64 IP requests, |U| = 512, 100 Zipf items),
configs[2] (64 requests, 200 items, lognormal |U|, larger-side rule -> mixed UP/IP), and small
mixed batches with RE requests, headers, ragged multi-page items, GQA groups 6 / 7 and d = 64."""
import numpy as np
import pytest

import synth
from oracle import plan as oplan

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

INT32_MIN = -2 ** 31


@pytest.fixture(scope="module")
def B():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
    bat.lib()
    return bat


def _dummy_model(cfg):
    """A bat_model with uninitialised device weights of the right shapes (planning does not read
    weight values)."""
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel
    H, F, d, Hq, Hkv, V = cfg["hidden"], cfg["ffn"], cfg["head_dim"], cfg["q_heads"], cfg["kv_heads"], cfg["vocab"]
    e = lambda *s: torch.empty(*s, dtype=torch.bfloat16, device="cuda")
    layers = [dict(ln1=e(H), wqkv=e((Hq + 2 * Hkv) * d, H), bqkv=e((Hq + 2 * Hkv) * d), wo=e(H, Hq * d),
                   ln2=e(H), wgu=e(2 * F, H), wd=e(H, F)) for _ in range(cfg["layers"])]
    emb = e(V, H)
    return DeviceModel(cfg, tensors=dict(embed=emb, lm_head=emb, final_norm=e(H), layers=layers))


def _reserve(B, pool, queries):
    ep = {}
    for q in queries:
        if not q.use_cache:
            continue
        if q.order == "UP":
            ents = [(B.BAT_ENT_USER, int(q.user_id), len(q.user_tok))]
        else:
            ents = [(B.BAT_ENT_HEADER, int(q.header_id), len(q.header_tok))] if len(q.header_tok) else []
            ents += [(B.BAT_ENT_ITEM, int(i), len(t)) for i, t in zip(q.item_ids, q.item_toks)]
        for kind, eid, n in ents:
            if (kind, eid) in ep:
                continue
            B.bat_kv_reserve(pool.handle, kind, eid, n)
            n_tok, pages = B.bat_kv_lookup(pool.handle, kind, eid)
            ep[(kind, eid)] = (list(pages), n_tok)
    return ep


def _check_batch(B, cfg, queries, n_pages):
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DevicePool
    model = _dummy_model(cfg)
    pool = DevicePool(cfg, n_pages)
    ep = _reserve(B, pool, queries)
    group = cfg["q_heads"] // cfg["kv_heads"]
    stream = torch.cuda.current_stream()
    plan = B.bat_plan_build(pool.handle, model.handle, B.QueryArray(queries), stream)
    n_listed = n_partial_rows = 0
    try:
        sp = 0
        qtile0 = 0
        for b, q in enumerate(queries):
            ref = oplan.plan_query(q, ep, group, sp)
            sp += (ref["S"] + 15) // 16
            S, qt = ref["S"], oplan.qtile_tokens(group)
            # the fused QKV epilogue's per-row destinations (row map -> q-tile, suffix page, slot)
            t = np.arange(S)
            want_st = np.stack([qtile0 + t // qt, ref["pages"][ref["n_prefix_pages"] + t // 16], t % 16], axis=1)
            got_st = B.bat_plan_export_device(plan, b, B.BAT_PFD_STAGE).reshape(S, 3)
            assert np.array_equal(got_st, want_st), (b, "a4 destinations", np.argwhere(got_st != want_st)[:5])
            qtile0 += (S + qt - 1) // qt
            n_kt = ref["tile_state"].shape[1]
            want = np.zeros((S, n_kt * 128), np.uint8)
            want[:, : ref["vis"].shape[1]] = ref["vis"]
            vis = B.bat_plan_export_device(plan, b, B.BAT_PFD_VIS).reshape(S, n_kt * 128)
            assert np.array_equal(vis, want), (b, q.order, np.argwhere(vis != want)[:5])
            last = B.bat_plan_export_device(plan, b, B.BAT_PFD_VIS_LAST).reshape(S, n_kt * 128)
            r0 = (ref["tile_state"].shape[0] - 1) * qt
            want_last = np.zeros_like(want)
            want_last[r0:] = want[r0:]
            assert np.array_equal(last, want_last), (b, "last layer")
            kp = B.bat_plan_export_device(plan, b, B.BAT_PFD_KPAGES).reshape(n_kt, 8)
            pages = np.full(n_kt * 8, INT32_MIN, np.int64)
            pages[: len(ref["pages"])] = ref["pages"]
            pages = pages.reshape(n_kt, 8)
            live = ref["tile_state"].max(axis=0) > 0
            for j in range(n_kt):
                if live[j]:
                    assert np.array_equal(kp[j], pages[j]), (b, j, kp[j], pages[j])
                else:
                    assert np.all(kp[j] == B.BAT_PFD_NOT_LOADED), (b, j, "dead tile loaded")
            n_listed += int(live.sum())
            n_partial_rows += int((ref["tile_state"] == 2).sum())
    finally:
        B.bat_plan_destroy(plan)
        pool.close()
        model.close()
    print(f"{len(queries)} requests: {n_listed} loaded k-tiles, {n_partial_rows} partial (q-tile, k-tile) pairs")
    assert n_partial_rows > 0  # the masks were exercised


def test_device_plan_config1_bench_batch(B):
    cfg = synth.model_config("qwen2-1.5b")
    rng = np.random.default_rng(7)
    zp = synth.zipf_weights(8192)
    qs = [synth.make_query(0, cfg, 1000 + b, 512, synth.distinct_label_items(0, cfg, 100, rng, 8192, zp),
                           (16, 16), 8, "IP") for b in range(64)]
    _check_batch(B, cfg, qs, 8192 + 64)


def test_device_plan_config2_mixed_batch(B):
    cfg = synth.model_config("qwen2-1.5b")
    rng = np.random.default_rng(11)
    zp = synth.zipf_weights(8192)
    n_user = synth.user_lengths(5, 64)
    qs = [synth.make_query(0, cfg, 5000 + b, int(n_user[b]),
                           synth.distinct_label_items(0, cfg, 200, rng, 8192, zp), (16, 16), 8,
                           "UP" if n_user[b] >= 200 * 16 else "IP") for b in range(64)]
    assert 0 < sum(q.order == "UP" for q in qs) < 64
    _check_batch(B, cfg, qs, 8192 + sum((len(q.user_tok) + 15) // 16 for q in qs) + 64)


@pytest.mark.parametrize("cfg_name", ["small", "small7", "small64", "tiny"])
def test_device_plan_small_mixed(B, cfg_name):
    cfg = synth.model_config(cfg_name)
    qs = [synth.make_query(4, cfg, 10 + i, n_u, list(range(50 + 3 * i, 62 + 3 * i)), (5, 37),
                           1 + i % 4, order, use_cache=(i != 3), n_header=(3 if i == 2 else 0))
          for i, (n_u, order) in enumerate([(40, "IP"), (250, "UP"), (8, "IP"), (60, "IP"), (130, "UP"),
                                            (0, "IP"), (300, "IP")])]
    _check_batch(B, cfg, qs, 2048)

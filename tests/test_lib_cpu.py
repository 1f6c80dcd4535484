"""CPU tests of the C-ABI library (no GPU): it loads, exports every symbol include/bat.h
declares, and its host logic (the planner, Algorithm 1, argument validation) matches the
oracle bit-exact.  The plan is built on an index-only pool (device = -1: no arena)."""
import os
import re

import numpy as np
import pytest

import synth
from oracle import hrcs as ohrcs
from oracle import plan as oplan

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "bat.h")


@pytest.fixture(scope="module")
def B():
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
    if not os.path.exists(bat.LIB_PATH):
        import __graft_entry__
        __graft_entry__.build()
    bat.lib()
    return bat


def test_exports_every_declared_symbol(B):
    decl = set(re.findall(r"BAT_API\s+[\w\s\*]+?\b(bat_\w+)\s*\(", open(HEADER).read()))
    assert len(decl) >= 25
    L = B.lib()
    for name in decl:
        assert hasattr(L, name), name
    assert set(decl) == set(B.EXPORTED)
    assert "sm_100a" in B.bat_version()


def _index_pool(B, cfg, n_pages=4096):
    return B.bat_kv_pool_create(-1, n_pages, cfg["layers"], cfg["kv_heads"], cfg["head_dim"])


def _reserve_for(B, pool, queries):
    """Reserve pages in the index-only pool for every prefix entry, in first-use order, and
    return the oracle's entity_pages map read back through bat_kv_lookup."""
    ep = {}
    for q in queries:
        ents = [(B.BAT_ENT_USER, q.user_id, len(q.user_tok))]
        if len(q.header_tok):
            ents.append((B.BAT_ENT_HEADER, q.header_id, len(q.header_tok)))
        ents += [(B.BAT_ENT_ITEM, int(i), len(t)) for i, t in zip(q.item_ids, q.item_toks)]
        for kind, eid, n in ents:
            if (kind, eid) in ep or n == 0:
                continue
            B.bat_kv_reserve(pool, kind, eid, n)
            n_tok, pages = B.bat_kv_lookup(pool, kind, eid)
            ep[(kind, eid)] = (list(pages), n_tok)
    return ep


def _compare_plan(B, plan, b, ref):
    info = B.bat_plan_query_info(plan, b)
    assert info["S"] == ref["S"] and info["P"] == ref["P"]
    assert info["n_prefix_pages"] == ref["n_prefix_pages"]
    assert info["n_live_pairs"] == ref["n_live_pairs"]
    assert info["scratch0"] == ref["scratch_page0"] and info["token_off"] == ref["token_off"]
    for field, key in [(B.BAT_PF_TOKENS, "tokens"), (B.BAT_PF_POS, "pos"), (B.BAT_PF_SEG, "seg"),
                       (B.BAT_PF_PAGES, "pages"), (B.BAT_PF_VALID, "valid"), (B.BAT_PF_KSEG, "kseg"),
                       (B.BAT_PF_KORD, "kord"), (B.BAT_PF_DISC, "disc")]:
        np.testing.assert_array_equal(B.bat_plan_export(plan, b, field), ref[key].astype(np.int32), err_msg=key)
    tiles = B.bat_plan_export(plan, b, B.BAT_PF_TILES).reshape(info["n_qtiles"], info["n_ktiles"])
    np.testing.assert_array_equal(tiles, ref["tile_state"])


@pytest.mark.parametrize("cfg_name,group", [("tiny", 2), ("small", 6)])
@pytest.mark.parametrize("seed", range(4))
def test_plan_bit_exact_vs_oracle(B, cfg_name, group, seed):
    cfg = synth.model_config(cfg_name)
    rng = np.random.default_rng(100 + seed)
    queries = []
    item_len = (int(rng.integers(1, 12)), int(rng.integers(12, 40)))  # one length per item id
    for k in range(4):
        order = ["UP", "IP", "IP", "RE"][k]
        n_items = int(rng.integers(1, 12))
        queries.append(synth.make_query(
            seed, cfg, user_id=int(rng.integers(0, 5)), n_user=int(rng.integers(0, 70)),
            item_ids=rng.choice(50, size=n_items, replace=False),
            item_len=item_len,
            n_instr=int(rng.integers(1, 9)), order="UP" if order == "UP" else "IP",
            use_cache=(order != "RE"), n_header=3 if (order == "IP" and seed % 2) else 0))
    # users must have one length per id: regenerate lengths per (user_id)
    lens = {}
    for q in queries:
        lens.setdefault(q.user_id, len(q.user_tok))
    queries = [synth.make_query(seed, cfg, q.user_id, lens[q.user_id], q.item_ids, item_len,
                                len(q.instr_tok), q.order, q.use_cache, len(q.header_tok)) for q in queries]
    pool = _index_pool(B, cfg)
    try:
        ep = _reserve_for(B, pool, queries)
        refs = oplan.plan_batch(queries, ep, group)
        plan = B.bat_plan_create(pool, group, B.QueryArray(queries))
        try:
            for b, ref in enumerate(refs):
                _compare_plan(B, plan, b, ref)
        finally:
            B.bat_plan_destroy(plan)
    finally:
        B.bat_kv_pool_destroy(pool)


def test_plan_qwen_shaped_single_query(B):
    """configs[1] shape: |U| = 512, 100 items x 16 tokens, IP and UP (group 6, 21-token q-tiles)."""
    cfg = synth.model_config("qwen2-1.5b")
    qs = [synth.make_query(0, cfg, 7, 512, list(range(100)), (16, 16), 8, o) for o in ("IP", "UP")]
    pool = _index_pool(B, cfg, 1024)
    try:
        ep = _reserve_for(B, pool, qs)
        refs = oplan.plan_batch(qs, ep, 6)
        plan = B.bat_plan_create(pool, 6, B.QueryArray(qs))
        try:
            for b, ref in enumerate(refs):
                _compare_plan(B, plan, b, ref)
            # live pairs per layer per head
            assert B.bat_plan_query_info(plan, 0)["n_live_pairs"] * 12 == 967460 * 12
        finally:
            B.bat_plan_destroy(plan)
    finally:
        B.bat_kv_pool_destroy(pool)


@pytest.mark.parametrize("seed", range(3))
def test_plan_multi_discriminant_rows_bit_exact(B, seed):
    """One discriminant per item: the planner's discriminant rows (the last suffix token
    of every item) equal the oracle plan's, for UP requests with cached or recomputed users and
    ragged items; IP is rejected."""
    cfg = synth.model_config("tiny")
    rng = np.random.default_rng(300 + seed)
    qs = []
    for k in range(3):
        q = synth.make_query(seed, cfg, user_id=k, n_user=int(rng.integers(1, 60)),
                             item_ids=rng.choice(40, size=int(rng.integers(1, 9)), replace=False),
                             item_len=(3, 21), n_instr=int(rng.integers(1, 5)), order="UP", use_cache=(k != 1))
        q.multi_disc = True
        qs.append(q)
    pool = _index_pool(B, cfg)
    try:
        ep = _reserve_for(B, pool, qs)
        refs = oplan.plan_batch(qs, ep, 2)
        plan = B.bat_plan_create(pool, 2, B.QueryArray(qs))
        try:
            for b, ref in enumerate(refs):
                _compare_plan(B, plan, b, ref)
                assert len(ref["disc"]) == qs[b].n_items
        finally:
            B.bat_plan_destroy(plan)
        bad = synth.make_query(seed, cfg, 0, qs[0].user_tok.size, qs[0].item_ids, (3, 21), 2, "IP")
        bad.multi_disc = True
        with pytest.raises(B.BatError):
            B.bat_plan_create(pool, 2, B.QueryArray([bad]))
    finally:
        B.bat_kv_pool_destroy(pool)


def test_missing_prefix_entry_is_notfound(B):
    cfg = synth.model_config("tiny")
    pool = _index_pool(B, cfg)
    try:
        q = synth.make_query(0, cfg, 1, 5, [1, 2], (4, 4), 1, "IP")
        with pytest.raises(B.BatError) as e:
            B.bat_plan_create(pool, 2, B.QueryArray([q]))
        assert e.value.status == -4
    finally:
        B.bat_kv_pool_destroy(pool)


def test_validation_errors(B):
    cfg = synth.model_config("tiny")
    pool = _index_pool(B, cfg)
    try:
        q = synth.make_query(0, cfg, 1, 5, [1, 2], (4, 4), 1, "IP", use_cache=False)
        q.instr_tok = np.zeros(0, np.int32)            # no discriminant token (reading R8)
        with pytest.raises(B.BatError) as e:
            B.bat_plan_create(pool, 2, B.QueryArray([q]))
        assert e.value.status == -1
        with pytest.raises(B.BatError):
            B.bat_kv_pool_create(-1, 16, 2, 2, 16, page_tokens=32)
        B.bat_kv_reserve(pool, B.BAT_ENT_ITEM, 9, 20)
        with pytest.raises(B.BatError):
            B.bat_kv_reserve(pool, B.BAT_ENT_ITEM, 9, 20)  # exists
        free0 = B.bat_kv_pool_stats(pool)[0]
        with pytest.raises(B.BatError) as e:
            B.bat_kv_reserve(pool, B.BAT_ENT_ITEM, 10, 16 * 5000)
        assert e.value.status == -5 and B.bat_kv_pool_stats(pool)[0] == free0  # all-or-nothing
        B.bat_kv_evict(pool, B.BAT_ENT_ITEM, 9)
        assert B.bat_kv_pool_stats(pool)[0] == free0 + 2
    finally:
        B.bat_kv_pool_destroy(pool)


@pytest.mark.parametrize("seed", range(5))
def test_hrcs_matches_oracle(B, seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(5, 300))
    F = rng.pareto(1.1, size=n) + 1e-3
    F[rng.integers(0, n, size=n // 5)] = F[0]  # ties
    for r_max in (0.0, 0.05, 0.3, 0.9, 1.0, 3.0):
        for world in (1, 2, 4, 8):
            r, owner = B.bat_hrcs_place(F, r_max, world)
            r_ref = ohrcs.replication_ratio(F, r_max)
            rep, own = ohrcs.place(F, r_ref, world)
            assert r == r_ref
            exp = np.array([-1 if i in set(rep) else own[i] for i in range(n)], dtype=np.int32)
            np.testing.assert_array_equal(owner, exp)
    assert B.bat_hrcs_rmax(100, 2, 0.1, 10, 5, 4) == pytest.approx(ohrcs.rmax_paper(100, 2, 0.1, 10, 5, 4), rel=1e-15)


@pytest.mark.parametrize("seed", range(5))
def test_hrcs_refresh_matches_oracle(B, seed):
    rng = np.random.default_rng(50 + seed)
    n_old = int(rng.integers(1, 300))
    n_new = n_old + int(rng.integers(0, 40))
    for world in (1, 2, 8):
        for r in (0.0, 0.1, 0.5, 1.0):
            F_old = rng.pareto(1.1, size=n_old) + 1e-3
            F_old[rng.integers(0, n_old, size=n_old // 4)] = F_old[0]  # ties
            rep, own = ohrcs.place(F_old, r, world)
            owner_old = [-1 if i in set(rep) else own[i] for i in range(n_old)]
            F_new = rng.pareto(1.1, size=n_new) + 1e-3
            F_new[rng.integers(0, n_new, size=n_new // 4)] = F_new[-1]
            got = B.bat_hrcs_refresh(owner_old, F_new, r, world)
            np.testing.assert_array_equal(got, np.array(ohrcs.refresh(owner_old, F_new, r, world), np.int32))


@pytest.mark.parametrize("seed", range(4))
def test_plan_pic_bit_exact_vs_oracle(B, seed):
    """Selective recompute (PIC, reading R25): item heads served from the cached entries (pages
    trimmed to |I| - k tokens), the tails recomputed after U — the C++ plan bit-exact against the
    oracle's plan over random ragged items, headers, RE and plain IP neighbours."""
    cfg = synth.model_config("tiny")
    rng = np.random.default_rng(300 + seed)
    item_len = (1, 37)
    queries = []
    for k in range(5):
        q = synth.make_query(seed, cfg, user_id=10 + k, n_user=int(rng.integers(0, 60)),
                             item_ids=rng.choice(40, size=int(rng.integers(1, 9)), replace=False),
                             item_len=item_len, n_instr=int(rng.integers(1, 5)), order="IP",
                             use_cache=(k != 4), n_header=3 if k == 2 else 0)
        q.pic_tail = [0, 1, 5, 17, 40][k]
        queries.append(q)
    pool = _index_pool(B, cfg)
    try:
        ep = _reserve_for(B, pool, queries)
        refs = oplan.plan_batch(queries, ep, 2)
        plan = B.bat_plan_create(pool, 2, B.QueryArray(queries))
        try:
            for b, ref in enumerate(refs):
                _compare_plan(B, plan, b, ref)
        finally:
            B.bat_plan_destroy(plan)
    finally:
        B.bat_kv_pool_destroy(pool)
    with pytest.raises(B.BatError):  # PIC is an Item-as-prefix notion
        q = synth.make_query(0, cfg, 1, 5, [1, 2], (4, 4), 1, "UP")
        q.pic_tail = 2
        pool = _index_pool(B, cfg)
        try:
            _reserve_for(B, pool, [q])
            B.bat_plan_create(pool, 2, B.QueryArray([q]))
        finally:
            B.bat_kv_pool_destroy(pool)

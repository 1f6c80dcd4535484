"""Single-GPU test of the cold-item pull (a10): two pools in one process stand in for two
ranks (bat_debug_attach_peer_pool maps the other arena as a peer, as CUDA IPC does across
processes).  The pulled pages must be byte-identical to the owner's, and a prefill served from
pulled items must give bit-identical hidden states to the same prefill on the owner's pool."""
import numpy as np
import pytest

import synth
from oracle import hrcs as ohrcs

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def B():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
    bat.lib()
    return bat


def test_cold_item_pull_is_bit_exact_and_serves_identically(B):
    from paper_conf_asplos_0017wzlxszh0w26_b200 import dist as bdist
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel, DevicePool
    cfg = synth.model_config("small")
    W = synth.Weights(cfg, seed=1)
    model = DeviceModel(cfg, W)
    owner_pool = DevicePool(cfg, 512, rank=1, world=2)   # rank 1 owns the items
    local_pool = DevicePool(cfg, 512, rank=0, world=2)   # rank 0 pulls them
    items = list(range(300, 330))
    toks = [synth.item_tokens(0, i, 16, cfg["vocab"]) for i in items]
    B.bat_kv_prefill_entities(owner_pool.handle, model.handle, B.BAT_ENT_ITEM, items, toks, 0)
    owner = np.full(400, -1, np.int32)
    owner[items] = 1
    for i in items:
        n_tok, pages = B.bat_kv_lookup(owner_pool.handle, B.BAT_ENT_ITEM, i)
        B.bat_kv_register_remote(local_pool.handle, B.BAT_ENT_ITEM, i, 1, pages, n_tok)
    B.bat_debug_attach_peer_pool(local_pool.handle, 1, owner_pool.handle)
    q = synth.make_query(0, cfg, 7, 50, items[:20], (16, 16), 4, "IP")
    cold = bdist.cold_items([q], owner, 0)
    assert list(cold) == sorted(items[:20])
    assert bdist.fetch_cold(local_pool.handle, cold) == 20
    assert bdist.fetch_cold(local_pool.handle, cold) == 0            # already local: one more reference
    L, Hkv, d = cfg["layers"], cfg["kv_heads"], cfg["head_dim"]
    for i in cold[:5]:
        ka = torch.empty(L, 16, Hkv, d, dtype=torch.bfloat16, device="cuda"); va = torch.empty_like(ka)
        kb = torch.empty_like(ka); vb = torch.empty_like(ka)
        B.bat_kv_read(owner_pool.handle, B.BAT_ENT_ITEM, int(i), ka, va)
        B.bat_kv_read(local_pool.handle, B.BAT_ENT_ITEM, int(i), kb, vb)
        assert torch.equal(ka, kb) and torch.equal(va, vb)
    h_owner = torch.empty(1, cfg["hidden"], device="cuda")
    h_local = torch.empty(1, cfg["hidden"], device="cuda")
    B.bat_bipartite_prefill(owner_pool.handle, model.handle, B.QueryArray([q]), h_owner)
    B.bat_bipartite_prefill(local_pool.handle, model.handle, B.QueryArray([q]), h_local)
    torch.cuda.synchronize()
    assert torch.equal(h_owner, h_local)
    bdist.release_cold(local_pool.handle, cold)                      # 2 references -> 1: still there
    B.bat_bipartite_prefill(local_pool.handle, model.handle, B.QueryArray([q]), h_local)
    bdist.release_cold(local_pool.handle, cold)                      # last reference: freed in stream order
    with pytest.raises(B.BatError):
        B.bat_bipartite_prefill(local_pool.handle, model.handle, B.QueryArray([q]), h_local)
    with pytest.raises(B.BatError):                                  # more releases than fetches
        bdist.release_cold(local_pool.handle, cold)
    local_pool.close(); owner_pool.close(); model.close()


def _two_pools(B, cfg, model, items, n_pages=2048):
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DevicePool
    owner_pool = DevicePool(cfg, n_pages, rank=1, world=2)
    local_pool = DevicePool(cfg, n_pages, rank=0, world=2)
    toks = [synth.item_tokens(0, i, 16, cfg["vocab"]) for i in items]
    for s in range(0, len(items), 256):
        B.bat_kv_prefill_entities(owner_pool.handle, model.handle, B.BAT_ENT_ITEM, items[s:s + 256], toks[s:s + 256], 0)
    for i in items:
        n_tok, pages = B.bat_kv_lookup(owner_pool.handle, B.BAT_ENT_ITEM, i)
        B.bat_kv_register_remote(local_pool.handle, B.BAT_ENT_ITEM, i, 1, pages, n_tok)
    B.bat_debug_attach_peer_pool(local_pool.handle, 1, owner_pool.handle)
    return owner_pool, local_pool


def _batches(cfg, items, n_batches, B_req=8, n_items=40, seed=3):
    rng = np.random.default_rng(seed)
    return [[synth.make_query(0, cfg, 100 * k + b, 200, rng.choice(items, n_items, replace=False), (16, 16), 4, "IP")
             for b in range(B_req)] for k in range(n_batches)]


def test_cold_pipeline_one_batch_ahead_overlaps_and_serves_identically(B):
    """ColdPipeline: batch k+1's pull runs on a copy stream while batch k computes; pages of
    released batches are reused behind stream waits.  Every batch's hidden states equal those of the
    same batch served from the owner's pool, and the event timeline shows the pulls inside compute."""
    from paper_conf_asplos_0017wzlxszh0w26_b200 import dist as bdist
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel
    cfg = synth.model_config("small")
    model = DeviceModel(cfg, synth.Weights(cfg, seed=1))
    items = list(range(1000, 1600))
    owner_pool, local_pool = _two_pools(B, cfg, model, items)
    batches = _batches(cfg, items, 6, B_req=24, n_items=24)  # compute long enough to hide a pull
    owner = np.full(2000, -1, np.int32)
    owner[items] = 1
    compute, copy = torch.cuda.current_stream(), torch.cuda.Stream()
    pipe = bdist.ColdPipeline(local_pool.handle, compute, copy)
    free0 = B.bat_kv_pool_stats(local_pool.handle)[0]
    outs, ev = [], []
    cold = [bdist.cold_items(b, owner, 0) for b in batches]
    t0 = torch.cuda.Event(enable_timing=True)
    t0.record(compute)
    pipe.prefetch(0, cold[0])
    qas = [B.QueryArray(qs) for qs in batches]
    for k, qs in enumerate(batches):
        pipe.acquire(k)
        c0 = torch.cuda.Event(enable_timing=True); c0.record(compute)
        h = torch.empty(len(qs), cfg["hidden"], device="cuda")
        B.bat_bipartite_prefill(local_pool.handle, model.handle, qas[k], h, compute)
        c1 = torch.cuda.Event(enable_timing=True); c1.record(compute)
        if k + 1 < len(batches):
            f0 = torch.cuda.Event(enable_timing=True); f0.record(copy)
            pipe.prefetch(k + 1, cold[k + 1])
            f1 = torch.cuda.Event(enable_timing=True); f1.record(copy)
        pipe.release(k)
        outs.append(h)
        ev.append((c0, c1) + ((f0, f1) if k + 1 < len(batches) else ()))
    torch.cuda.synchronize()
    assert B.bat_kv_pool_stats(local_pool.handle)[0] == free0  # every pulled page given back
    overlapped = 0
    for k in range(len(batches) - 1):
        c0, c1, f0, f1 = ev[k]
        a, b, fa, fb = t0.elapsed_time(c0), t0.elapsed_time(c1), t0.elapsed_time(f0), t0.elapsed_time(f1)
        overlapped += int(fa < b and fb > a)  # the pull of k+1 intersects the compute of k
        print(f"batch {k}: compute [{a:.3f}, {b:.3f}] ms, pull of {k + 1} [{fa:.3f}, {fb:.3f}] ms")
    assert overlapped >= len(batches) - 2
    for qs, h in zip(batches, outs):
        ref = torch.empty_like(h)
        B.bat_bipartite_prefill(owner_pool.handle, model.handle, B.QueryArray(qs), ref)
        torch.cuda.synchronize()
        assert torch.equal(h, ref)
    local_pool.close(); owner_pool.close(); model.close()


def test_staged_plans_double_buffered_serve_identically(B):
    """Pre-built plans with staged cold items (bat_plan_build_staged, 2 slots): the pull of batch
    k+1 into slot (k+1)%2 waits for batch k-1 (same slot) and overlaps batch k; outputs equal the
    owner-pool plans bit for bit, across two passes over the batches."""
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel
    cfg = synth.model_config("small")
    model = DeviceModel(cfg, synth.Weights(cfg, seed=1))
    items = list(range(2000, 2600))
    owner_pool, local_pool = _two_pools(B, cfg, model, items)
    B.bat_kv_staging_reserve(local_pool.handle, 2, 8 * 40)
    batches = _batches(cfg, items, 4, seed=5)
    compute, copy = torch.cuda.current_stream(), torch.cuda.Stream()
    plans = [B.bat_plan_build_staged(local_pool.handle, model.handle, B.QueryArray(qs), k % 2, compute)
             for k, qs in enumerate(batches)]
    ref_plans = [B.bat_plan_build(owner_pool.handle, model.handle, B.QueryArray(qs), compute) for qs in batches]
    refs = []
    for p, qs in zip(ref_plans, batches):
        h = torch.empty(len(qs), cfg["hidden"], device="cuda")
        B.bat_prefill_plan(owner_pool.handle, model.handle, p, h, compute)
        refs.append(h)
    n_steps = 8
    fetched = [None] * (n_steps + 1)
    done = [None] * n_steps
    def pull(i):
        if i >= 2:
            copy.wait_event(done[i - 2])  # the slot's previous reader has finished
        n = B.bat_plan_fetch(local_pool.handle, plans[i % 4], copy)
        e = torch.cuda.Event(); e.record(copy)
        fetched[i] = e
        return n
    assert pull(0) > 0
    outs = []
    for i in range(n_steps):
        if i + 1 < n_steps:
            pull(i + 1)
        compute.wait_event(fetched[i])
        h = torch.empty(len(batches[i % 4]), cfg["hidden"], device="cuda")
        B.bat_prefill_plan(local_pool.handle, model.handle, plans[i % 4], h, compute)
        done[i] = torch.cuda.Event(); done[i].record(compute)
        outs.append(h)
    torch.cuda.synchronize()
    for i, h in enumerate(outs):
        assert torch.equal(h, refs[i % 4]), i
    with pytest.raises(B.BatError):  # plans built on another pool are refused
        B.bat_prefill_plan(local_pool.handle, model.handle, ref_plans[0], outs[0], compute)
    for p in plans + ref_plans:
        B.bat_plan_destroy(p)
    local_pool.close(); owner_pool.close(); model.close()


def test_plan_pins_entries_until_destroyed(B):
    """A pre-built plan's device image holds page ids: evicting an entry it reads is refused
    (BAT_E_STATE) until the plan is destroyed; destroying the pool first is refused too."""
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel, DevicePool, prefill_missing_entities
    cfg = synth.model_config("tiny")
    model = DeviceModel(cfg, synth.Weights(cfg, seed=1))
    pool = DevicePool(cfg, 256)
    q = synth.make_query(0, cfg, 3, 16, [11, 22, 33, 44], (8, 8), 2, "IP")
    prefill_missing_entities(pool, model, [q])
    plan = B.bat_plan_build(pool.handle, model.handle, B.QueryArray([q]))
    with pytest.raises(B.BatError) as e:
        B.bat_kv_evict(pool.handle, B.BAT_ENT_ITEM, 22)
    assert e.value.status == -7
    with pytest.raises(B.BatError):
        B.bat_kv_pool_destroy(pool.handle)
    B.bat_plan_destroy(plan)
    B.bat_kv_evict(pool.handle, B.BAT_ENT_ITEM, 22)
    pool.close(); model.close()


def test_placement_refresh_and_new_items_serve_identically(B):
    """NEXT-1 (P:312 Step 3, footnote P:322): after a burst changes item hotness and new items
    join the corpus, bat_hrcs_refresh's placement is applied on both 'ranks' (two pools on one
    GPU): promoted items pulled into the replicated area, demoted ones dropped by non-owners, new
    items computed by their owner.  Requests over old and new items then serve bit-identically
    to a pool that computed every item itself, before and after the refresh."""
    from paper_conf_asplos_0017wzlxszh0w26_b200 import dist as bdist
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel, DevicePool
    cfg = synth.model_config("small")
    model = DeviceModel(cfg, synth.Weights(cfg, seed=1))
    tok = lambda i: synth.item_tokens(0, int(i), 16, cfg["vocab"])
    n_old, n_new, r = 60, 70, 0.2
    F = synth.zipf_weights(n_old)
    rep, own = ohrcs.place(F, r, 2)
    owner = np.array([-1 if i in set(rep) else own[i] for i in range(n_old)], np.int32)
    pools = [DevicePool(cfg, 1024, rank=k, world=2) for k in range(2)]
    for k in range(2):
        B.bat_debug_attach_peer_pool(pools[k].handle, 1 - k, pools[1 - k].handle)
        mine = bdist.local_items(owner, k)
        B.bat_kv_prefill_entities(pools[k].handle, model.handle, B.BAT_ENT_ITEM, mine, [tok(i) for i in mine], 0)

    def register(owner_vec):
        for k in range(2):
            for i in np.nonzero(owner_vec == 1 - k)[0]:
                n_tok, pages = B.bat_kv_lookup(pools[1 - k].handle, B.BAT_ENT_ITEM, int(i))
                B.bat_kv_register_remote(pools[k].handle, B.BAT_ENT_ITEM, int(i), 1 - k, pages, n_tok)

    register(owner)
    ref_pool = DevicePool(cfg, 1024)
    B.bat_kv_prefill_entities(ref_pool.handle, model.handle, B.BAT_ENT_ITEM, list(range(n_new)),
                              [tok(i) for i in range(n_new)], 0)

    def serve_and_compare(owner_vec, items_range):
        rng = np.random.default_rng(9)
        for k in range(2):
            qs = [synth.make_query(0, cfg, 40 + b, 30, rng.choice(items_range, 12, replace=False), (16, 16), 2, "IP")
                  for b in range(3)]
            cold = bdist.cold_items(qs, owner_vec, k)
            bdist.fetch_cold(pools[k].handle, cold)
            h = torch.empty(3, cfg["hidden"], device="cuda")
            ref = torch.empty_like(h)
            B.bat_bipartite_prefill(pools[k].handle, model.handle, B.QueryArray(qs), h)
            B.bat_bipartite_prefill(ref_pool.handle, model.handle, B.QueryArray(qs), ref)
            bdist.release_cold(pools[k].handle, cold, torch.cuda.current_stream())
            torch.cuda.synchronize()
            assert torch.equal(h, ref)

    serve_and_compare(owner, np.arange(n_old))
    F_new = np.concatenate([F, np.full(n_new - n_old, F[3])])
    F_new[[40, 50, 55]] = F.max() * 2  # burst hotspots
    owner_new = bdist.refresh_placement(owner, F_new, r, 2)
    np.testing.assert_array_equal(owner_new, np.array(ohrcs.refresh(list(owner), F_new, r, 2), np.int32))
    assert owner[40] >= 0 and owner_new[40] == -1  # a cold item promoted by the burst
    moves = [bdist.apply_refresh(pools[k].handle, model.handle, owner, owner_new, k, tok) for k in range(2)]
    assert sum(m["promoted"] for m in moves) > 0 and sum(m["computed"] for m in moves) >= n_new - n_old
    register(owner_new)
    for k in range(2):  # every item is stored where the new placement says
        for i in range(n_new):
            local = owner_new[i] < 0 or owner_new[i] == k
            try:
                B.bat_kv_lookup(pools[k].handle, B.BAT_ENT_ITEM, i)
                assert local, (k, i)
            except B.BatError:
                assert not local, (k, i)
    serve_and_compare(owner_new, np.arange(n_new))
    for p_ in pools + [ref_pool]:
        p_.close()
    model.close()


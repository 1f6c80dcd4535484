"""Single-GPU test of the cold-item pull (a10): two pools in one process stand in for two
ranks (bat_debug_attach_peer_pool maps the other arena as a peer, as CUDA IPC does across
processes).  The pulled pages must be byte-identical to the owner's, and a prefill served from
pulled items must give bit-identical hidden states to the same prefill on the owner's pool."""
import numpy as np
import pytest

import synth

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
    assert bdist.fetch_cold(local_pool.handle, cold) == 0            # already local: dedup
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
    bdist.drop_fetched(local_pool.handle, cold)
    with pytest.raises(B.BatError):
        B.bat_bipartite_prefill(local_pool.handle, model.handle, B.QueryArray([q]), h_local)
    local_pool.close(); owner_pool.close(); model.close()

"""Multi-process CPU tests (torch.distributed gloo, world size 2) of the data-parallel host
logic: Algorithm 1 placement identical on every rank, owned sets disjoint and complete,
remote page tables registered exactly as the owners hold them, per-batch cold-item dedup,
and request load balancing.  Pools are index-only (device = -1): no GPU needed."""
import os
import socket

import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, ret):
    import torch.distributed as dist
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat, dist as bdist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        cfg = synth.model_config("tiny")
        corpus = 400
        freq = synth.zipf_weights(corpus)
        r, owner = bdist.place_items(freq, 0.5, world)
        pool = bat.bat_kv_pool_create(-1, 4096, cfg["layers"], cfg["kv_heads"], cfg["head_dim"],
                                      rank=rank, world=world)
        mine = bdist.local_items(owner, rank)
        for i in mine:
            bat.bat_kv_reserve(pool, bat.BAT_ENT_ITEM, i, 8 + i % 20)
        n_remote = bdist.exchange_remote(pool, owner, rank, world, attach_ipc=False)
        # page tables as registered here vs as the owners hold them
        regs = {}
        for i in np.nonzero((owner >= 0) & (owner != rank))[0]:
            o, n_tok, pages = bat.bat_kv_lookup_remote(pool, bat.BAT_ENT_ITEM, int(i))
            regs[int(i)] = (o, n_tok, [int(p) for p in pages])
        held = {i: bat.bat_kv_lookup(pool, bat.BAT_ENT_ITEM, i) for i in mine}
        held = {i: (n, [int(p) for p in pg]) for i, (n, pg) in held.items()}
        owners = [None] * world
        dist.all_gather_object(owners, owner.tolist())
        helds = [None] * world
        dist.all_gather_object(helds, held)
        rng = np.random.default_rng(rank)
        qs = [synth.make_query(0, cfg, u, 5, rng.choice(corpus, 12, replace=False, p=freq), (4, 4), 1, "IP")
              for u in range(6)]
        cold = bdist.cold_items(qs, owner, rank)
        ret[rank] = dict(r=r, owners=owners, regs=regs, helds=helds, n_remote=n_remote, mine=mine,
                         cold=cold.tolist(), items=[q.item_ids.tolist() for q in qs])
        bat.bat_kv_pool_destroy(pool)
    finally:
        dist.destroy_process_group()


def test_two_rank_placement_and_remote_registration():
    import torch.multiprocessing as mp
    world = 2
    mgr = mp.Manager()
    ret = mgr.dict()
    mp.spawn(_worker, args=(world, _free_port(), ret), nprocs=world, join=True)
    res = [ret[r] for r in range(world)]
    # identical placement on every rank
    assert res[0]["owners"][0] == res[0]["owners"][1] == res[1]["owners"][0]
    owner = np.array(res[0]["owners"][0])
    assert res[0]["r"] == res[1]["r"]
    rep = set(np.nonzero(owner < 0)[0].tolist())
    # owned sets disjoint, together with the replicas they cover the corpus
    s0 = set(res[0]["mine"]) - rep
    s1 = set(res[1]["mine"]) - rep
    assert not (s0 & s1) and (s0 | s1 | rep) == set(range(len(owner)))
    assert abs(len(s0) - len(s1)) <= 1                           # round-robin by hotness rank
    for rank in range(world):
        other = 1 - rank
        regs = res[rank]["regs"]
        assert res[rank]["n_remote"] == len(regs) == len(set(res[other]["mine"]) - rep)
        for i, (o, n_tok, pages) in regs.items():
            assert o == other
            assert (n_tok, pages) == tuple(res[other]["helds"][other][i])
        # cold-item dedup: every needed non-local item exactly once, sorted
        want = sorted({i for items in res[rank]["items"] for i in items if owner[i] >= 0 and owner[i] != rank})
        assert res[rank]["cold"] == want


def test_partition_requests_balanced():
    from paper_conf_asplos_0017wzlxszh0w26_b200 import dist as bdist
    rng = np.random.default_rng(0)
    lens = list(rng.integers(100, 8000, size=64))
    parts = bdist.partition_requests(lens, 8)
    assert sorted(i for p in parts for i in p) == list(range(64))
    loads = [sum(lens[i] for i in p) for p in parts]
    assert max(loads) - min(loads) <= max(lens)

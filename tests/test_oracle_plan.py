"""Pins for oracle/plan.py: a hand-checked small plan, and the plan's key-slot visibility
cross-checked against the explicit sequence mask of oracle/sequence.py (two independent
formulations of P:249-257 must agree on every pair)."""
import numpy as np
import pytest

import synth
from oracle import plan as op
from oracle.sequence import build_sequence, bipartite_mask

CFG = synth.model_config("tiny")


def _pages_for(queries, start=0):
    """Allocate pool pages for every prefix entity the way a fresh pool would: in order of
    first appearance, ceil(n/16) consecutive page ids each."""
    pages, nxt = {}, start
    for q in queries:
        ents = []
        ents.append(((op.ENT_USER, q.user_id), len(q.user_tok)))
        if len(q.header_tok):
            ents.append(((op.ENT_HEADER, q.header_id), len(q.header_tok)))
        for iid, t in zip(q.item_ids, q.item_toks):
            ents.append(((op.ENT_ITEM, int(iid)), len(t)))
        for key, n in ents:
            if key not in pages:
                np_ = (n + 15) // 16
                pages[key] = (list(range(nxt, nxt + np_)), n)
                nxt += np_
    return pages


def test_hand_checked_ip_plan():
    q = synth.make_query(0, CFG, 7, 3, [5, 6], (16, 16), 1, "IP")
    ep = {(op.ENT_USER, 7): ([0], 3), (op.ENT_ITEM, 5): ([1], 16), (op.ENT_ITEM, 6): ([2], 16)}
    p = op.plan_query(q, ep, group=2)
    assert p["P"] == 32 and p["S"] == 4
    assert list(p["pos"]) == [16, 17, 18, 19]           # U at m + p, Instr after U
    assert list(p["seg"]) == [-1, -1, -1, -2]
    assert list(p["pages"]) == [1, 2, -1]               # item pages, then scratch page 0
    assert list(p["valid"]) == [16, 16, 4]
    assert list(p["kseg"][:32]) == [0] * 16 + [1] * 16
    assert list(p["kord"][:36]) == [0] * 32 + [1, 2, 3, 4]
    assert all(p["kord"][36:] == op.INVALID_ORD)
    # one q-tile (64 tokens fit), one k-tile of 48 slots: suffix causal -> partial
    assert p["tile_state"].tolist() == [[2]]
    assert p["n_live_pairs"] == 4 * 32 + (1 + 2 + 3 + 4)


def test_hand_checked_up_plan_skip_and_full():
    # UP, group 6 -> 21 tokens per q-tile; user of 128 tokens = 8 pages = exactly k-tile 0
    cfg = dict(CFG, q_heads=12, kv_heads=2)
    q = synth.make_query(0, cfg, 1, 128, list(range(10, 20)), (16, 16), 1, "UP")
    ep = {(op.ENT_USER, 1): (list(range(100, 108)), 128)}
    p = op.plan_query(q, ep, group=6)
    assert p["S"] == 161
    st = p["tile_state"]
    assert st.shape == (8, 3)
    assert (st[:, 0] == 1).all()                        # every row sees the whole user: full
    # q-tile 0 = item0 tokens 0..15 + item1 tokens 0..4; k-tile 2 = suffix slots 96..160
    # (items 6..9 + instr): invisible to items 0/1 -> skip
    assert st[0, 2] == 0
    assert st[7, 2] == 2                                 # last tile holds the Instr row


@pytest.mark.parametrize("order", ["UP", "IP", "RE"])
@pytest.mark.parametrize("seed", range(6))
def test_plan_visibility_equals_sequence_mask(order, seed):
    rng = np.random.default_rng(seed)
    n_items = int(rng.integers(1, 6))
    q = synth.make_query(seed, CFG, 3, int(rng.integers(0, 40)), list(range(n_items)),
                         (int(rng.integers(1, 10)), int(rng.integers(10, 24))),
                         int(rng.integers(1, 4)), "UP" if order == "UP" else "IP",
                         use_cache=(order != "RE"), n_header=int(seed % 2) * 3 if order == "IP" else 0)
    ep = _pages_for([q])
    p = op.plan_query(q, ep, group=2)
    toks, seg, pos = build_sequence(q.order, q.user_tok, q.item_toks, q.instr_tok,
                                    q.header_tok if q.order == "IP" else ())
    M = bipartite_mask(seg)
    P, S = p["P"], p["S"]
    assert np.array_equal(p["tokens"], toks[P:]) and np.array_equal(p["pos"], pos[P:])
    # map every valid key slot to its index in the full sequence
    slot_to_seq = []
    seq_i = 0
    for pi, nv in enumerate(p["valid"]):
        for j in range(16):
            slot_to_seq.append(seq_i + j if j < nv else -1)
        seq_i += nv
    slot_to_seq = np.array(slot_to_seq)
    assert seq_i == P + S
    vis = (p["kord"][None, :] <= p["rord"][:, None]) & (
        (p["kseg"][None, :] == p["seg"][:, None]) | (p["kseg"][None, :] < 0) | (p["seg"][:, None] < 0))
    for t in range(S):
        for k, sq in enumerate(slot_to_seq):
            want = bool(M[P + t, sq]) if sq >= 0 else False
            assert vis[t, k] == want
    assert p["n_live_pairs"] == int(M[P:, :].sum())


def test_plan_batch_offsets():
    qs = [synth.make_query(0, CFG, u, 5 + u, [1, 2], (16, 16), 2, "IP") for u in range(3)]
    ps = op.plan_batch(qs, _pages_for(qs), group=2)
    assert [p["token_off"] for p in ps] == [0, 7, 15]
    assert [p["scratch_page0"] for p in ps] == [0, 1, 2]


@pytest.mark.parametrize("seed", range(3))
def test_multi_disc_rows_by_position(seed):
    """The plan's per-item discriminant rows (R20), by a second formulation: item i's
    discriminant is the suffix row of segment i whose POSITION is |U| + |I_i| - 1 (items
    start at position |U| in UP; positions are pinned by tests/golden/mask_tiny.txt)."""
    cfg = synth.model_config("tiny")
    q = synth.make_query(seed, cfg, 2, 7 + seed, [3, 1, 4, 5][: 2 + seed], (2, 11), 2, "UP", use_cache=(seed != 1))
    q.multi_disc = True
    p = op.plan_query(q, _pages_for([q]), 2)
    for i, t in enumerate(q.item_toks):
        rows = np.nonzero((p["seg"] == i) & (p["pos"] == len(q.user_tok) + len(t) - 1))[0]
        assert len(rows) == 1 and p["disc"][i] == rows[0]

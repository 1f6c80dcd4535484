"""Pins for the selective-recompute variant of Item-as-prefix (PAPER.md P:265
"position-independent caching ... selectively recomputes some critical tokens", "PIC like
CacheBlend ... narrowing the gap between IP and UP"; reading DESIGN.md R25).

PIC(k): every item's last k tokens are recomputed per request AFTER the user tokens (they attend to
the header, their own item's cached head, U and their own earlier tail tokens; never another
item), at positions continuing after U.  Pinned by:
  * k = 0 is exactly IP (the same prompt);
  * with no header and k >= max |I_i| every item token is recomputed after U: the UP prompt
    shifted by m positions, so PIC == UP up to RoPE's relative-position invariance (1e-9 in fp64)
    — the two orderings the paper compares are the end points of PIC;
  * hand-written order / segments / positions of a tiny prompt;
  * cached heads == full recompute (I1), permutation equivariance (I3), item independence of the
    cached heads (I2; the tails depend on the other items through U, by construction)."""
import numpy as np
import pytest

import synth
from oracle import model as om
from oracle.sequence import HEADER, INSTR, USER, bipartite_mask, build_sequence

CFG = synth.model_config("tiny")


@pytest.fixture(scope="module")
def W():
    return synth.Weights(CFG, seed=1)


def _q(order="IP", pic=0, items=(11, 22, 33, 44), n_user=12, item_len=(3, 9), n_header=0, seed=0):
    q = synth.make_query(seed, CFG, 3, n_user, list(items), item_len, 2, order, n_header=n_header)
    q.pic_tail = pic
    return q


def test_pic_hand_written_order_segments_positions():
    U, I1, I2, X = [7, 8], [1, 2, 3], [4, 5], [9]
    toks, seg, pos = build_sequence("IP", U, [I1, I2], X, (), pic_tail=1)
    # [I1 head (2), I2 head (1), U, I1 tail, I2 tail, X]; m = 3, |U| = 2
    assert list(toks) == [1, 2, 4, 7, 8, 3, 5, 9]
    assert list(seg) == [0, 0, 1, USER, USER, 0, 1, INSTR]
    assert list(pos) == [0, 1, 0, 3, 4, 2 + 5, 1 + 5, 8]
    M = bipartite_mask(seg)
    assert M[5, 0] and M[5, 1] and M[5, 3] and M[5, 4] and not M[5, 2]  # I1 tail: own head + U, not I2
    assert M[6, 2] and not M[6, 5] and not M[6, 0]                       # I2 tail: own head, not I1
    assert M[7].all()                                                    # Instr sees everything


def test_pic_zero_is_ip(W):
    a = om.run_query(CFG, W, _q("IP", 0), "full")
    b = om.run_query(CFG, W, _q("IP", 0), "cached")
    q = _q("IP", 0)
    q.pic_tail = 0
    t0 = build_sequence("IP", q.user_tok, q.item_toks, q.instr_tok)
    t1 = build_sequence("IP", q.user_tok, q.item_toks, q.instr_tok, (), 0)
    assert all(np.array_equal(x, y) for x, y in zip(t0, t1))
    np.testing.assert_allclose(a["s"], b["s"], rtol=1e-10, atol=1e-12)


def test_pic_full_recompute_equals_up(W):
    """k >= m, no header: the prompt is UP's shifted by m positions -> the same scores."""
    up = om.run_query(CFG, W, _q("UP"), "full")
    pic = om.run_query(CFG, W, _q("IP", pic=9), "full")
    np.testing.assert_allclose(pic["hf"], up["hf"], rtol=1e-9, atol=1e-9)
    np.testing.assert_allclose(pic["z"], up["z"], rtol=1e-9, atol=1e-9)
    ip = om.run_query(CFG, W, _q("IP"), "full")
    assert np.max(np.abs(ip["z"] - up["z"])) > 1e-3  # and IP itself differs (reading R1)


@pytest.mark.parametrize("k", [1, 2, 5])
def test_pic_cached_heads_equal_full_recompute(W, k):
    """I1: serving the heads from the items' standalone KV (first |I| - k rows) == recomputing
    the whole PIC prompt."""
    for n_header in (0, 3):
        a = om.run_query(CFG, W, _q("IP", k, n_header=n_header), "full")
        b = om.run_query(CFG, W, _q("IP", k, n_header=n_header), "cached")
        np.testing.assert_allclose(a["hf"], b["hf"], rtol=1e-10, atol=1e-10)


def test_pic_permutation_equivariance(W):
    a = om.run_query(CFG, W, _q("IP", 2, items=(11, 22, 33, 44)), "full")
    b = om.run_query(CFG, W, _q("IP", 2, items=(33, 11, 44, 22)), "full")
    np.testing.assert_allclose(b["s"], a["s"][[2, 0, 3, 1]], rtol=1e-9, atol=1e-12)


def test_pic_item_independence(W):
    """I2 for the cached part: every item's head (the tokens still served from the cache) never
    depends on another item's tokens.  The recomputed tails attend to U, and U (in IP order)
    attends to every item's head, so a tail DOES depend on the other items — through U only."""
    q1 = _q("IP", 2)
    q2 = _q("IP", 2)
    q2.item_toks = list(q2.item_toks)
    q2.item_toks[1] = (np.asarray(q2.item_toks[1]) + 5) % CFG["vocab"]
    outs = []
    for q in (q1, q2):
        toks, seg, pos = build_sequence("IP", q.user_tok, q.item_toks, q.instr_tok, (), 2)
        h, _ = om.forward_full(CFG, W, toks, pos, bipartite_mask(seg))
        n_head = sum(len(t) - min(2, len(t)) for t in q.item_toks)
        outs.append((h, seg, n_head))
    (h1, s1, n1), (h2, s2, n2) = outs
    assert n1 == n2
    for item in (0, 2, 3):
        heads = np.nonzero(s1[:n1] == item)[0]
        np.testing.assert_allclose(h1[heads], h2[heads], rtol=1e-12, atol=1e-12)
        tails = np.nonzero(s1 == item)[0]
        tails = tails[tails >= n1]
        assert np.max(np.abs(h1[tails] - h2[tails])) > 1e-6  # through U

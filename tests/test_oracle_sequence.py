"""Pins for oracle/sequence.py: hand-written golden masks (tests/golden/mask_tiny.txt) and
brute-force statements of P:249-257 on random tiny prompts."""
import os

import numpy as np
import pytest

from oracle.sequence import build_sequence, bipartite_mask, HEADER, INSTR, USER

GOLD = os.path.join(os.path.dirname(__file__), "golden", "mask_tiny.txt")


def _read_golden():
    out, cur = {}, None
    for line in open(GOLD):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        if line.startswith("["):
            cur = line[1:-1]
            out[cur] = dict(rows=[])
            continue
        parts = line.split()
        if parts[0] == "order":
            out[cur]["order"] = parts[1:]
        elif parts[0] == "pos":
            out[cur]["pos"] = [int(x) for x in parts[1:]]
        else:
            out[cur]["rows"].append([int(x) for x in parts[1:]])
    return out


@pytest.mark.parametrize("order", ["UP", "IP"])
def test_golden_tiny_mask_and_positions(order):
    g = _read_golden()[order]
    U, I1, I2, X = [100, 101], [200, 201], [300], [400]
    toks, seg, pos = build_sequence(order, U, [I1, I2], X)
    name = {100: "u0", 101: "u1", 200: "a0", 201: "a1", 300: "b0", 400: "x0"}
    assert [name[t] for t in toks] == g["order"]
    assert list(pos) == g["pos"]
    assert bipartite_mask(seg).astype(int).tolist() == g["rows"]


def _random_prompt(rng, order, hdr=0):
    nu = int(rng.integers(0, 6))
    n = int(rng.integers(1, 5))
    items = [list(rng.integers(0, 50, size=int(rng.integers(1, 5)))) for _ in range(n)]
    X = list(rng.integers(0, 50, size=int(rng.integers(1, 3))))
    U = list(rng.integers(0, 50, size=nu))
    H = list(rng.integers(0, 50, size=hdr)) if order == "IP" else []
    return U, items, X, H


@pytest.mark.parametrize("order", ["UP", "IP"])
@pytest.mark.parametrize("seed", range(20))
def test_brute_force_rules(order, seed):
    rng = np.random.default_rng(seed)
    U, items, X, H = _random_prompt(rng, order, hdr=int(seed % 3) if order == "IP" else 0)
    toks, seg, pos = build_sequence(order, U, items, X, H)
    M = bipartite_mask(seg)
    T = len(toks)
    m = max(len(t) for t in items)
    # expected index ranges of each segment, written out from the prompt orders P:249/P:253
    idx = {}
    cur = 0
    segs_in_order = (["U"] + [("I", i) for i in range(len(items))] + ["X"]) if order == "UP" \
        else (["H"] + [("I", i) for i in range(len(items))] + ["U", "X"])
    sizes = {"U": len(U), "X": len(X), "H": len(H)}
    for s in segs_in_order:
        n = len(items[s[1]]) if isinstance(s, tuple) else sizes[s]
        idx[s] = list(range(cur, cur + n))
        cur += n
    assert cur == T
    # all items share one starting position: |U| (UP) or h (IP, after the header)
    start = len(U) if order == "UP" else len(H)
    for i in range(len(items)):
        assert [pos[t] for t in idx[("I", i)]] == [start + j for j in range(len(items[i]))]
    # reading R2: the segment after the items continues from start + m
    after = idx["X"] if order == "UP" else idx["U"] + idx["X"]
    assert [pos[t] for t in after] == [start + m + j for j in range(len(after))]
    for q in range(T):
        for k in range(T):
            both_items = seg[q] >= 0 and seg[k] >= 0
            # P:257 / P:131: different items never see each other
            if both_items and seg[q] != seg[k]:
                assert not M[q, k]
            elif k <= q:
                assert M[q, k]  # causal otherwise (R5); users/instr see items and vice versa (R4)
            else:
                assert not M[q, k]
    # each item is independent of later user and instruction tokens
    for i in range(len(items)):
        for q in idx[("I", i)]:
            visible = set(np.nonzero(M[q])[0])
            allowed = set(idx.get("U", []) if order == "UP" else []) | set(idx.get("H", [])) | set(idx[("I", i)])
            assert visible <= allowed


def test_segment_ids():
    toks, seg, pos = build_sequence("IP", [1, 2], [[3], [4, 5]], [6], header_tok=[7])
    assert list(seg) == [HEADER, 0, 1, 1, USER, USER, INSTR]
    assert list(pos) == [0, 1, 1, 2, 3, 4, 5]

"""Prompt scheduler + user-prefix cache: the C++
scheduler of libbat (host bookkeeping, no GPU) against the plain reference simulation in
oracle/scheduler.py — every decision (order, hit, evicted users) and every total must match
exactly on synthetic long-tail traces, for all five policies."""
import pytest

import synth
from oracle import scheduler as osched


@pytest.fixture(scope="module")
def B():
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
    bat.lib()
    return bat


def _run_lib(B, trace, policy, cap, window):
    s = B.bat_sched_create(policy, cap, window)
    out = []
    for (t, u, tu, ti) in trace:
        order, hit, admit, ev, f = B.bat_sched_decide(s, t, u, tu, ti)
        out.append((order, hit, ev))
    st = B.bat_sched_stats(s)
    B.bat_sched_destroy(s)
    return out, st


@pytest.mark.parametrize("policy", osched.POLICIES)
@pytest.mark.parametrize("cap", [0, 300, 3000, 30000])
def test_scheduler_matches_reference_simulation(B, policy, cap):
    trace = synth.request_trace(7, 3000, 400, rate=20.0)
    ref, rtot = osched.simulate(trace, policy, cap, window=30.0)
    got, gtot = _run_lib(B, trace, policy, cap, 30.0)
    for k, (a, b) in enumerate(zip(got, ref)):
        assert a == b, (k, trace[k], a, b)
    for key in ("tokens", "reused", "hits", "up", "ip"):
        assert gtot[key] == rtot[key], key
    assert gtot["used_pages"] <= cap


def test_scheduler_hand_trace(B):
    """Hand-checked trace (capacity 700 pages = 11,200 tokens; W = 10): u1 (250 pages) and u2
    (313) fit; u3 (375, f=1) may not evict u2 (f=1, not lower) -> IP; u4 is shorter than the
    items -> IP; u3 again (f=2) evicts u2 (f=1) -> UP."""
    tr = [(0.0, 1, 4000, 1600), (1.0, 2, 5000, 1600), (2.0, 1, 4000, 1600), (3.0, 3, 6000, 1600),
          (3.5, 4, 500, 1600), (4.0, 3, 6000, 1600)]
    got, st = _run_lib(B, tr, "hotness", 700, 10.0)
    assert got == [("UP", False, []), ("UP", False, []), ("UP", True, []), ("IP", False, []),
                   ("IP", False, []), ("UP", False, [2])]
    assert st["reused"] == 4000 + 1600 + 1600 and st["hits"] == 1


def test_scheduler_rejects_time_going_backwards(B):
    s = B.bat_sched_create("hotness", 100, 5.0)
    B.bat_sched_decide(s, 2.0, 1, 100, 50)
    with pytest.raises(B.BatError):
        B.bat_sched_decide(s, 1.0, 1, 100, 50)
    B.bat_sched_destroy(s)

"""CUDA-graph replay of bat_prefill_plan (include/bat.h, opt-in BAT_GRAPH=1): a plan's first call on a capturable
stream sizes the workspace, the second captures the layer loop into a graph, later calls replay
it.  Replays must be bit-identical to the eager first call, re-capture after the workspace was
reallocated by a larger plan, count the same kernel launches, and match the fp64 oracle
(PAPER.md P:173-183 via tests/test_gpu_parity._check)."""
import numpy as np
import pytest

import synth
from tests import test_gpu_parity as G

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def B():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
    bat.lib()
    return bat


def test_prefill_plan_graph_replay_is_bit_identical(B, monkeypatch):
    monkeypatch.setenv("BAT_GRAPH", "1")  # opt-in, read by every bat_prefill_plan call
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DevicePool, prefill_missing_entities
    cfg, W, model = G._model("small")
    pool = DevicePool(cfg, 4096)
    small = [synth.make_query(3, cfg, 40 + i, 60 + 30 * i, list(range(100 + 4 * i, 112 + 4 * i)), (5, 19), 2,
                              "IP" if i % 2 else "UP") for i in range(3)]
    big = [synth.make_query(4, cfg, 60 + i, 400, list(range(300, 340)), (16, 16), 8, "IP") for i in range(6)]
    prefill_missing_entities(pool, model, small + big)
    st = torch.cuda.Stream()
    plan = B.bat_plan_build(pool.handle, model.handle, B.QueryArray(small), st)
    plan_big = B.bat_plan_build(pool.handle, model.handle, B.QueryArray(big), st)
    outs, launches = [], []
    hidden = torch.empty(len(small), cfg["hidden"], device="cuda")
    hidden_big = torch.empty(len(big), cfg["hidden"], device="cuda")
    for i in range(6):
        if i == 3:  # a larger batch grows the shared workspace: the next call must not replay
            B.bat_prefill_plan(pool.handle, model.handle, plan_big, hidden_big, st)
        hidden.fill_(float("nan"))
        st.synchronize()
        n0 = B.bat_kernel_launch_count()
        B.bat_prefill_plan(pool.handle, model.handle, plan, hidden, st)
        launches.append(B.bat_kernel_launch_count() - n0)
        st.synchronize()
        outs.append(hidden.cpu().numpy().copy())
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])
    assert len(set(launches)) == 1 and launches[0] > 0, launches
    # the replayed output is the prefill the oracle defines (scores from the same hidden states)
    n_max = max(q.n_items for q in small)
    labels = np.zeros((len(small), n_max), np.int32)
    for b, q in enumerate(small):
        labels[b, : q.n_items] = q.labels
    lab = torch.tensor(labels, device="cuda")
    nit = torch.tensor([q.n_items for q in small], dtype=torch.int32, device="cuda")
    scores = torch.empty(len(small), n_max, device="cuda")
    logits = torch.empty(len(small), n_max, device="cuda")
    topk = torch.empty(len(small), 3, dtype=torch.int32, device="cuda")
    B.bat_score(model.handle, hidden, lab, nit, len(small), n_max, scores, 3, topk, logits=logits)
    torch.cuda.synchronize()
    out = dict(hf=hidden.double().cpu().numpy(), s=scores.double().cpu().numpy(),
               z=logits.double().cpu().numpy(), topk=topk.cpu().numpy())
    G._check(cfg, W, small, out)
    B.bat_plan_destroy(plan)
    B.bat_plan_destroy(plan_big)
    pool.close()

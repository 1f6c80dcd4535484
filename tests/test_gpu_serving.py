"""End-to-end serving with the prompt scheduler on the GPU: the hotness-aware
and greedy policies decide each request's prefix side, the user cache is admitted / evicted in
the pool, and every served request must still equal the oracle's full recompute of the prompt in
the order the scheduler chose (2e-2 abs/rel on hf and s)."""
import numpy as np
import pytest

import synth
from oracle import model as om
from tests.gpu_util import max_excess

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.mark.parametrize("policy", ["hotness", "greedy"])
def test_trace_serving_matches_oracle(policy):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel, DevicePool, TraceServer
    cfg = synth.model_config("tiny")
    W = synth.Weights(cfg, seed=1)
    model = DeviceModel(cfg, W)
    pool = DevicePool(cfg, 512)
    rng = np.random.default_rng(5)
    # 4 candidates x 8 tokens = 32 item tokens; users of 20..60 tokens (2..4 pages); user cache of
    # 6 pages: admissions, hits, hotness-based refusals and evictions all occur
    lens = {u: int(x) for u, x in zip(range(6), [20, 60, 45, 12, 33, 50])}
    users = [0, 1, 0, 2, 1, 3, 4, 0, 5, 1, 2, 0, 4, 4, 5, 1]
    reqs = []
    for i, u in enumerate(users):
        items = synth.distinct_label_items(1, cfg, 4, rng, 64)
        reqs.append((float(i), u, lens[u], items))
    srv = TraceServer(pool, model, policy, user_capacity_pages=6, window=6.0, seed=1, n_instr=2, item_len=(8, 8))
    batches = srv.serve(reqs, batch=4)
    torch.cuda.synchronize()
    orders = [d[0] for d in srv.decisions]
    assert "UP" in orders and "IP" in orders
    if policy == "hotness":
        assert any(d[1] for d in srv.decisions)  # at least one user-cache hit
    worst = -1.0
    for qs, hidden, scores in batches:
        hf = hidden.double().cpu().numpy()
        s = scores.double().cpu().numpy()
        for b, q in enumerate(qs):
            ref = om.run_query(cfg, W, q, "full")
            worst = max(worst, max_excess(hf[b], ref["hf"]), max_excess(s[b, : q.n_items], ref["s"]))
    print(policy, orders, srv.stats(), "worst excess", worst)
    assert worst <= 0
    srv.close()
    pool.close()
    model.close()

"""Multi-discriminant variant ("one discriminant token per item"; SURVEY §8(f) NEXT-3;
DESIGN.md R20) through the C ABI: bat_bipartite_prefill with multi_disc writes one final hidden
state per item (its last token), bat_score_multi scores item i against its own row.  Checked
against oracle.model.run_query_multi (full recompute): 2e-2 abs/rel in bf16, 1e-5 in the fp32
mode, on hf, z and s."""
import numpy as np
import pytest

import synth
from oracle import model as om
from tests.gpu_util import max_excess

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def B():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
    bat.lib()
    return bat


_MODELS = {}


def _model(name, dtype):
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel
    if (name, dtype) not in _MODELS:
        cfg = synth.model_config(name)
        W = synth.Weights(cfg, seed=1)
        _MODELS[(name, dtype)] = (cfg, W, DeviceModel(cfg, W, dtype=dtype))
    return _MODELS[(name, dtype)]


def _queries(cfg, name):
    if name == "tiny":
        specs = [(0, 3, 40, [11, 22, 33, 44], (8, 8), 2, True), (1, 4, 50, [5, 6, 7], (6, 12), 3, False)]
    else:
        specs = [(3, 6, 300, list(range(200, 220)), (16, 16), 8, True), (4, 7, 200, list(range(60, 72)), (10, 16), 4, False)]
    qs = []
    for seed, uid, nu, items, il, ni, cache in specs:
        q = synth.make_query(seed, cfg, uid, nu, items, il, ni, "UP", use_cache=cache)
        q.multi_disc = True
        qs.append(q)
    return qs


@pytest.mark.parametrize("name,dtype,tol", [("tiny", "bf16", 2e-2), ("small", "bf16", 2e-2),
                                            ("tiny", "fp32", 1e-5), ("small", "fp32", 1e-5)])
def test_multi_discriminant_matches_oracle(B, name, dtype, tol):
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DevicePool, prefill_missing_entities
    cfg, W, model = _model(name, dtype)
    qs = _queries(cfg, name)
    pool = DevicePool(cfg, 2048, dtype=dtype)
    prefill_missing_entities(pool, model, qs)
    Bn, n_max, H = len(qs), max(q.n_items for q in qs), cfg["hidden"]
    hidden = torch.empty(Bn, n_max, H, device="cuda")
    B.bat_bipartite_prefill(pool.handle, model.handle, B.QueryArray(qs), hidden)
    labels = np.zeros((Bn, n_max), np.int32)
    for b, q in enumerate(qs):
        labels[b, : q.n_items] = q.labels
    scores = torch.empty(Bn, n_max, device="cuda")
    B.bat_score_multi(model.handle, hidden, torch.tensor(labels, device="cuda"),
                      torch.tensor([q.n_items for q in qs], dtype=torch.int32, device="cuda"), Bn, n_max, scores)
    torch.cuda.synchronize()
    hf, s = hidden.double().cpu().numpy(), scores.double().cpu().numpy()
    worst = -1.0
    for b, q in enumerate(qs):
        ref = om.run_query_multi(cfg, W, q, "full")
        n = q.n_items
        z = np.einsum("ij,ij->i", np.asarray(W.lm_head_rows(q.labels), np.float64), hf[b, :n])
        for got, want in ((hf[b, :n], ref["hf"]), (z, ref["z"]), (s[b, :n], ref["s"])):
            worst = max(worst, max_excess(got, want, tol, tol))
    print(name, dtype, "worst excess", worst)
    assert worst <= 0
    pool.close()


def test_multi_discriminant_rejects_ip_and_mixed_batches(B):
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DevicePool
    cfg, W, model = _model("tiny", "bf16")
    pool = DevicePool(cfg, 256)
    q = synth.make_query(0, cfg, 3, 16, [11, 22], (8, 8), 2, "IP")
    q.multi_disc = True
    hidden = torch.empty(1, 2, cfg["hidden"], device="cuda")
    with pytest.raises(B.BatError):
        B.bat_bipartite_prefill(pool.handle, model.handle, B.QueryArray([q]), hidden)
    a = synth.make_query(0, cfg, 3, 40, [11, 22], (8, 8), 2, "UP", use_cache=False)
    b = synth.make_query(0, cfg, 4, 40, [11, 22], (8, 8), 2, "UP", use_cache=False)
    a.multi_disc = True
    with pytest.raises(B.BatError):
        B.bat_bipartite_prefill(pool.handle, model.handle, B.QueryArray([a, b]), hidden)
    pool.close()

"""Full-size GPU parity (B200) at BASELINE.json's shapes, in the launch configuration bench.py
times (bat_plan_build + bat_prefill_plan + bat_score over a whole batch), checked on SAMPLED
requests against the fp64 oracle's full recompute (the plain definition, oracle/model.py).

* configs[1]: Qwen2-1.5B shape, 28 layers, batch of 64 IP requests of |U| = 512 + 100 x
  16-token Zipf items + 8 instruction tokens (bench.py's step); requests 0 and 63 checked.
* configs[2]: Qwen2-1.5B shape, 200 candidates, batch of 64 with lognormal |U| and the
  larger-side prefix rule (UP iff |U| >= 200 x 16) — one IP and one UP request checked.
* configs[4]'s layer shape: Qwen2-7B width (hidden 3584, 28 Q / 4 KV heads, g = 7), 2 layers,
  |U| = 2048 + 200 items (IP), checked on every request of a batch of 2.
Tolerance (north_star, R11): |gpu - ref| <= 2e-2 + 2e-2 |ref| on hf, z and s.

Init (R12): MLP matrices N(0, 0.01^2), everything else N(0, 0.02^2).  With N(0, 0.02^2)
MLPs an IDEAL bf16 pipeline already misses the tolerance on hf after 28 layers (relative error
3%, tools/bf16_emulation_full.py: excess +0.07; this GPU path: +0.046) — bf16 rounding, not a
kernel bug; at 0.01 the ideal pipeline stays inside it (excess -0.007) while a wrong (plain
causal) mask still moves z by far more than 10x atol (asserted below, tools/mask_guard_full.py)."""
import numpy as np
import pytest

import synth
from oracle import model as om
from oracle.sequence import causal_mask
from tests.gpu_util import max_excess, score_excess

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def B():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
    bat.lib()
    return bat


_W = {}


def _weights(cfg, seed):
    """Generate each layer once and keep it (the oracle and the upload both read it)."""
    key = (cfg["hidden"], cfg["layers"], cfg.get("mlp_std"), seed)
    if key not in _W:
        W = synth.Weights(cfg, seed=seed)
        for l in range(cfg["layers"]):
            W._cache[l] = W.layer(l)
        _W[key] = W
    return _W[key]


def _serve_batch(B, cfg, W, queries, n_pages, k=10):
    """bench.py's launch configuration: pre-built device plan + bat_prefill_plan + bat_score."""
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import (DeviceModel, DevicePool,
                                                                prefill_missing_entities)
    model = DeviceModel(cfg, W)
    pool = DevicePool(cfg, n_pages)
    stream = torch.cuda.current_stream()
    prefill_missing_entities(pool, model, queries, stream=stream)
    Bn = len(queries)
    n_max = max(q.n_items for q in queries)
    qa = B.QueryArray(queries)
    plan = B.bat_plan_build(pool.handle, model.handle, qa, stream)
    hidden = torch.empty(Bn, cfg["hidden"], device="cuda")
    labels = np.zeros((Bn, n_max), np.int32)
    for b, q in enumerate(queries):
        labels[b, : q.n_items] = q.labels
    lab = torch.tensor(labels, device="cuda")
    nit = torch.tensor([q.n_items for q in queries], dtype=torch.int32, device="cuda")
    scores = torch.empty(Bn, n_max, device="cuda")
    logits = torch.empty(Bn, n_max, device="cuda")
    topk = torch.empty(Bn, k, dtype=torch.int32, device="cuda")
    # twice: the second pass must reproduce the first bit for bit (no state leaks between steps)
    outs = []
    for _ in range(2):
        B.bat_prefill_plan(pool.handle, model.handle, plan, hidden, stream)
        B.bat_score(model.handle, hidden, lab, nit, Bn, n_max, scores, k, topk, stream, logits=logits)
        torch.cuda.synchronize()
        outs.append((hidden.clone(), scores.clone(), topk.clone()))
    assert torch.equal(outs[0][0], outs[1][0]) and torch.equal(outs[0][2], outs[1][2])
    out = dict(hf=hidden.double().cpu().numpy(), s=scores.double().cpu().numpy(),
               z=logits.double().cpu().numpy(), topk=topk.cpu().numpy())
    B.bat_plan_destroy(plan)
    pool.close()
    model.close()
    return out


def _check_sampled(cfg, W, queries, out, sample, k=10):
    worst = {}
    for b in sample:
        q = queries[b]
        ref = om.run_query(cfg, W, q, "full", k=k)
        hf = out["hf"][b]
        z = out["z"][b, : q.n_items]  # the score kernel's own logits
        s = out["s"][b, : q.n_items]
        for name, got, want in (("hf", hf, ref["hf"]), ("z", z, ref["z"]), ("s", s, ref["s"])):
            worst[name] = max(worst.get(name, -1.0), max_excess(got, want))
        worst["log_s"] = max(worst.get("log_s", -1.0), score_excess(z, s, ref["z"], ref["s"])[1])
        srt = np.sort(ref["s"])[::-1]
        for r in range(k):  # top-k agrees wherever the oracle's rank margin exceeds the tolerance
            if r + 1 < len(srt) and srt[r] - srt[r + 1] > 2 * (2e-2 + 2e-2 * srt[r]):
                assert out["topk"][b, r] == ref["topk"][r], (b, r)
            else:
                break
        assert np.all(np.isfinite(out["s"][b, : q.n_items]))
        assert abs(out["s"][b, : q.n_items].sum() - 1.0) < 1e-4
    print("sampled", list(sample), "worst excess over tolerance:", {k: round(v, 5) for k, v in worst.items()})
    for name, v in worst.items():
        assert v <= 0, (name, v)


def _qwen(name):
    cfg = synth.model_config(name)
    cfg["mlp_std"] = 0.01  # full-size parity init (module docstring, R12)
    return cfg


def test_config1_bench_batch_sampled(B):
    """configs[1] exactly as bench.py serves it (batch 64, IP, Zipf items from 8,192)."""
    cfg = _qwen("qwen2-1.5b")
    W = _weights(cfg, 1)
    rng = np.random.default_rng(7)
    zp = synth.zipf_weights(8192)
    qs = [synth.make_query(0, cfg, 1000 + b, 512, synth.distinct_label_items(0, cfg, 100, rng, 8192, zp),
                           (16, 16), 8, "IP") for b in range(64)]
    out = _serve_batch(B, cfg, W, qs, n_pages=8192 + 64)
    _check_sampled(cfg, W, qs, out, [0, 63])
    # mask-sensitivity guard at this init and shape: a plain causal mask must be detectable
    good = om.run_query(cfg, W, qs[0], "full")
    bad = om.run_query(cfg, W, qs[0], "full", mask_fn=lambda seg: causal_mask(len(seg)))
    assert np.abs(good["z"] - bad["z"]).max() > 10 * 2e-2


def test_config2_mixed_batch_sampled(B):
    """configs[2]: 200 candidates, batch 64, lognormal |U|, larger-side prefix rule."""
    cfg = _qwen("qwen2-1.5b")
    W = _weights(cfg, 1)
    rng = np.random.default_rng(11)
    zp = synth.zipf_weights(8192)
    n_user = synth.user_lengths(5, 64)
    qs = []
    for b in range(64):
        order = "UP" if n_user[b] >= 200 * 16 else "IP"
        qs.append(synth.make_query(0, cfg, 5000 + b, int(n_user[b]),
                                   synth.distinct_label_items(0, cfg, 200, rng, 8192, zp), (16, 16), 8, order))
    n_up = sum(q.order == "UP" for q in qs)
    assert 0 < n_up < 64
    pages = 8192 + sum((len(q.user_tok) + 15) // 16 for q in qs if q.order == "UP") + 64
    out = _serve_batch(B, cfg, W, qs, n_pages=pages)
    ip = [b for b, q in enumerate(qs) if q.order == "IP"]
    up = [b for b, q in enumerate(qs) if q.order == "UP"]
    # the shortest UP request and a mid-length IP request keep the oracle's cost in bounds
    up_b = min(up, key=lambda b: len(qs[b].user_tok))
    ip_b = sorted(ip, key=lambda b: len(qs[b].user_tok))[len(ip) // 2]
    _check_sampled(cfg, W, qs, out, [ip_b, up_b])


def test_qwen7b_width_two_layers(B):
    """Qwen2-7B layer shape (hidden 3584, 28/4 heads: g = 7 packs 18 tokens x 7 heads per
    q-tile), |U| = 2048 + 200 x 16-token items, IP (configs[4]'s request), 2 layers."""
    cfg = _qwen("qwen2-7b")
    cfg["layers"] = 2
    # at hidden 3584 an ideal bf16 pipeline with N(0, 0.01^2) MLPs already misses the tolerance
    # after 2 layers (excess +0.028, tools/bf16_emulation_full.py); N(0, 0.005^2): -0.0067
    cfg["mlp_std"] = 0.005
    W = _weights(cfg, 3)
    rng = np.random.default_rng(13)
    qs = [synth.make_query(1, cfg, 77 + b, 2048, synth.distinct_label_items(1, cfg, 200, rng, 4096),
                           (16, 16), 8, "IP") for b in range(2)]
    out = _serve_batch(B, cfg, W, qs, n_pages=512)
    _check_sampled(cfg, W, qs, out, [0, 1])
    good = om.run_query(cfg, W, qs[0], "full")  # mask-sensitivity guard at this init and shape
    bad = om.run_query(cfg, W, qs[0], "full", mask_fn=lambda seg: causal_mask(len(seg)))
    assert np.abs(good["z"] - bad["z"]).max() > 10 * 2e-2

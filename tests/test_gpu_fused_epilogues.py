"""Fused epilogues.  (1) RMSNorm fused across the residual updates (a3 / a7): at batch sizes where no
projection takes the split-K path, the O and down GEMMs write h_new = h + acc, xg = bf16(h_new * g)
and per-N-tile sums of squares, and the QKV / gate-up GEMMs scale their rows by
rsqrt(mean(h^2) + eps) — the standalone norm kernel is not launched.  Both paths are checked
against the fp64 oracle's full recompute (2e-2 abs/rel on hf, z, s; R11) and against
each other; the launch count proves which path ran (2L - 1 norm launches fewer when fused).
(2) a4 (RoPE + q-tile / suffix-page staging) fused into the QKV GEMM epilogue (default for batches
whose QKV projection is not split-K): the same checks, L stage launches fewer."""
import os

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


def _queries(cfg, n, n_user, seed=7):
    rng = np.random.default_rng(seed)
    qs = []
    for b in range(n):
        items = rng.choice(5000, size=20, replace=False) + 1 + 100000 * b  # header or not: own items
        order = "UP" if b % 4 == 3 else "IP"
        qs.append(synth.make_query(seed, cfg, 100 + b, n_user + 37 * b, items, (9, 16), 8, order,
                                   n_header=(4 if b % 2 and order == "IP" else 0)))
    return qs


def _prefill(B, cfg, W, model, queries, fused, var="BAT_FUSED_NORM"):
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DevicePool, prefill_missing_entities
    pool = DevicePool(cfg, 8192)
    prefill_missing_entities(pool, model, queries)
    hidden = torch.empty(len(queries), cfg["hidden"], device="cuda")
    old = os.environ.get(var)
    os.environ[var] = fused if isinstance(fused, str) else ("1" if fused else "0")
    try:
        torch.cuda.synchronize()
        n0 = B.bat_kernel_launch_count()
        B.bat_bipartite_prefill(pool.handle, model.handle, B.QueryArray(queries), hidden)
        torch.cuda.synchronize()
        n = B.bat_kernel_launch_count() - n0
    finally:
        if old is None:
            del os.environ[var]
        else:
            os.environ[var] = old
    pool.close()
    return hidden.double().cpu().numpy(), n


@pytest.mark.parametrize("cfg_name,mode", [("small", "1"), ("small7", "1"), ("small", "d"), ("small7", "d")])
def test_fused_norm_matches_oracle_and_unfused(B, cfg_name, mode):
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel
    cfg = synth.model_config(cfg_name)
    W = synth.Weights(cfg, seed=3)
    model = DeviceModel(cfg, W)
    # ~4,300 suffix rows: every projection's tile grid fills the SMs (no split-K) -> fused path
    qs = _queries(cfg, 10, 420)
    hf_f, n_f = _prefill(B, cfg, W, model, qs, mode)
    hf_u, n_u = _prefill(B, cfg, W, model, qs, False)
    L = cfg["layers"]
    # the fused run skipped the norm kernels: ln1 of every layer (d), and ln2 of all but the last (1)
    assert n_u - n_f == (2 * L - 1 if mode == "1" else L), (n_u, n_f)
    # the two paths differ only by where bf16 rounds (h*g vs h*rstd*g) and the fp32 order of rstd
    assert max_excess(hf_f, hf_u, atol=1e-2, rtol=1e-2) <= 0.0
    worst = -1.0
    for b, q in enumerate(qs):
        ref = om.run_query(cfg, W, q, "full", k=1)
        worst = max(worst, max_excess(hf_f[b], ref["hf"]), max_excess(hf_u[b], ref["hf"]))
    assert worst <= 0.0, worst
    model.close()


def test_small_batch_keeps_standalone_norm(B):
    """Batch-1 shapes take split-K projections; the fused path is off there (same launches as
    BAT_FUSED_NORM=0) and the result is unchanged."""
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel
    cfg = synth.model_config("small")
    W = synth.Weights(cfg, seed=3)
    model = DeviceModel(cfg, W)
    qs = _queries(cfg, 1, 200)
    hf_f, n_f = _prefill(B, cfg, W, model, qs, True)
    hf_u, n_u = _prefill(B, cfg, W, model, qs, False)
    assert n_f == n_u
    assert np.array_equal(hf_f, hf_u)
    ref = om.run_query(cfg, W, qs[0], "full", k=1)
    assert max_excess(hf_f[0], ref["hf"]) <= 0.0
    model.close()


@pytest.mark.parametrize("cfg_name", ["small", "small7", "small64"])
def test_fused_stage_matches_oracle_and_unfused(B, cfg_name):
    """QKV epilogue staging (bias + RoPE in fp32, one bf16 rounding, q-tile / page stores) vs
    the separate stage kernel (bf16 qkv, then RoPE): both within the oracle tolerance, each other
    at 1e-2, and exactly L stage launches apart.  small7: 11 heads of 128 (a half-empty last
    N-tile); small64: d = 64 (four heads per N-tile)."""
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel
    cfg = synth.model_config(cfg_name)
    W = synth.Weights(cfg, seed=5)
    model = DeviceModel(cfg, W)
    qs = _queries(cfg, 10, 420, seed=11)
    hf_f, n_f = _prefill(B, cfg, W, model, qs, True, "BAT_FUSED_STAGE")
    hf_u, n_u = _prefill(B, cfg, W, model, qs, False, "BAT_FUSED_STAGE")
    assert n_u - n_f == cfg["layers"], (n_u, n_f)
    assert max_excess(hf_f, hf_u, atol=1e-2, rtol=1e-2) <= 0.0
    worst = -1.0
    for b, q in enumerate(qs):
        ref = om.run_query(cfg, W, q, "full", k=1)
        worst = max(worst, max_excess(hf_f[b], ref["hf"]), max_excess(hf_u[b], ref["hf"]))
    assert worst <= 0.0, worst
    model.close()


def test_fused_stage_entity_pages_and_no_stray_writes(B):
    """Entity precompute (the prefix-miss path writes the new entries' K/V straight into pool pages)
    on a batch large enough for the fused QKV-epilogue staging: the pages match the stage-kernel
    path within two bf16 roundings (1e-2), and an unrelated entry appended beforehand stays
    byte-identical in both pools (no stray 16-byte stores from the epilogue's scattered writes)."""
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel, DevicePool, prefill_missing_entities
    cfg = synth.model_config("small")
    W = synth.Weights(cfg, seed=9)
    model = DeviceModel(cfg, W)
    L, Hkv, d = cfg["layers"], cfg["kv_heads"], cfg["head_dim"]
    g = torch.Generator(device="cpu").manual_seed(4)
    ck = torch.randn(L, 37, Hkv, d, generator=g).to(torch.bfloat16).cuda()
    cv = torch.randn(L, 37, Hkv, d, generator=g).to(torch.bfloat16).cuda()
    qs = [synth.make_query(13, cfg, 500 + b, 64, np.arange(20) + 1 + 20 * b, (16, 16), 8, "IP") for b in range(12)]
    kv = {}
    for fused in (True, False):
        pool = DevicePool(cfg, 8192)
        B.bat_kv_append(pool.handle, B.BAT_ENT_USER, 999999, ck, cv, 37)
        old = os.environ.get("BAT_FUSED_STAGE")
        os.environ["BAT_FUSED_STAGE"] = "1" if fused else "0"
        try:
            prefill_missing_entities(pool, model, qs)  # 240 items x 16 tokens per entity call
            torch.cuda.synchronize()
        finally:
            if old is None:
                del os.environ["BAT_FUSED_STAGE"]
            else:
                os.environ["BAT_FUSED_STAGE"] = old
        ko = torch.empty(L, 37, Hkv, d, dtype=torch.bfloat16, device="cuda")
        vo = torch.empty_like(ko)
        B.bat_kv_read(pool.handle, B.BAT_ENT_USER, 999999, ko, vo)
        torch.cuda.synchronize()
        assert torch.equal(ko, ck) and torch.equal(vo, cv), f"canary entry changed (fused={fused})"
        items = {}
        for iid in range(1, 241):
            k = torch.empty(L, 16, Hkv, d, dtype=torch.bfloat16, device="cuda")
            v = torch.empty_like(k)
            B.bat_kv_read(pool.handle, B.BAT_ENT_ITEM, iid, k, v)
            items[iid] = (k.float().cpu().numpy(), v.float().cpu().numpy())
        kv[fused] = items
        pool.close()
    worst = max(max(max_excess(kv[True][i][j], kv[False][i][j], atol=1e-2, rtol=1e-2) for j in (0, 1))
                for i in kv[True])
    assert worst <= 0.0, worst
    model.close()

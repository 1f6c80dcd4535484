"""Kernel-level GPU parity (B200): the tcgen05 GEMM epilogues against an fp32 matmul of the
same bf16 operands; the KV page scatter/gather round trip (bit-exact); one layer of the
tcgen05 bipartite attention (stage + paged attention) against the fp64 oracle attention with
an explicit mask."""
import numpy as np
import pytest

import synth
from tests.gpu_util import max_excess, oracle_attention_layer, prefix_entities_in_order

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def B():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
    bat.lib()
    return bat


def _rand(shape, scale, seed):
    g = torch.Generator(device="cpu").manual_seed(seed)
    return (torch.randn(*shape, generator=g) * scale).to(torch.bfloat16).cuda()


GEMM_SHAPES = [(1, 64, 64), (37, 128, 64), (130, 256, 128), (300, 768, 1024), (520, 2048, 1536),
               (1000, 1536, 1536), (257, 512, 8960)]


@pytest.mark.parametrize("M,N,K", GEMM_SHAPES)
def test_gemm_bias_bf16(B, M, N, K):
    A, W, bias = _rand((M, K), 1.0, 1), _rand((N, K), 0.05, 2), _rand((N,), 0.1, 3)
    out = torch.empty(M, N, dtype=torch.bfloat16, device="cuda")
    B.bat_debug_gemm(1, M, N, K, A, W, N, out, N, bias)
    torch.cuda.synchronize()
    ref = A.float() @ W.float().T + bias.float()
    assert max_excess(out.float().cpu().numpy(), ref.cpu().numpy(), 1e-2, 1e-2) <= 0


@pytest.mark.parametrize("M,N,K", GEMM_SHAPES)
def test_gemm_residual_f32(B, M, N, K):
    A, W = _rand((M, K), 1.0, 4), _rand((N, K), 0.05, 5)
    h0 = torch.randn(M, N, device="cuda")
    out = h0.clone()
    B.bat_debug_gemm(2, M, N, K, A, W, N, out, N)
    torch.cuda.synchronize()
    ref = h0 + A.float() @ W.float().T
    assert max_excess(out.cpu().numpy(), ref.cpu().numpy(), 1e-3, 1e-3) <= 0


@pytest.mark.parametrize("M,F,K", [(5, 128, 64), (200, 1024, 768), (520, 8960, 1536)])
def test_gemm_swiglu(B, M, F, K):
    A, W = _rand((M, K), 1.0, 6), _rand((2 * F, K), 0.05, 7)
    out = torch.empty(M, F, dtype=torch.bfloat16, device="cuda")
    B.bat_debug_gemm(3, M, F, K, A, W, 2 * F, out, F, None, F)
    torch.cuda.synchronize()
    gu = A.float() @ W.float().T
    ref = torch.nn.functional.silu(gu[:, :F]) * gu[:, F:]
    assert max_excess(out.float().cpu().numpy(), ref.cpu().numpy(), 1e-2, 1e-2) <= 0


@pytest.mark.parametrize("cfg_name", ["tiny", "small"])
def test_kv_append_read_roundtrip_bit_exact(B, cfg_name):
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DevicePool
    cfg = synth.model_config(cfg_name)
    L, Hkv, d = cfg["layers"], cfg["kv_heads"], cfg["head_dim"]
    pool = DevicePool(cfg, 64)
    k1, v1 = _rand((L, 21, Hkv, d), 1.0, 8), _rand((L, 21, Hkv, d), 1.0, 9)
    k2, v2 = _rand((L, 30, Hkv, d), 1.0, 10), _rand((L, 30, Hkv, d), 1.0, 11)
    B.bat_kv_append(pool.handle, B.BAT_ENT_USER, 5, k1, v1, 21)
    B.bat_kv_append(pool.handle, B.BAT_ENT_USER, 5, k2, v2, 30)   # extends the last page
    n, pages = B.bat_kv_lookup(pool.handle, B.BAT_ENT_USER, 5)
    assert n == 51 and len(pages) == 4
    ko = torch.empty(L, 51, Hkv, d, dtype=torch.bfloat16, device="cuda")
    vo = torch.empty_like(ko)
    B.bat_kv_read(pool.handle, B.BAT_ENT_USER, 5, ko, vo)
    torch.cuda.synchronize()
    assert torch.equal(ko, torch.cat([k1, k2], 1)) and torch.equal(vo, torch.cat([v1, v2], 1))
    pool.close()


def _attention_case(B, cfg_name, queries_fn, layer=1, seed=0):
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel, DevicePool
    cfg = synth.model_config(cfg_name)
    W = synth.Weights(cfg, seed=seed)
    model = DeviceModel(cfg, W)
    pool = DevicePool(cfg, 2048)
    queries = queries_fn(cfg)
    L, Hkv, d = cfg["layers"], cfg["kv_heads"], cfg["head_dim"]
    ekv = {}
    for q in queries:
        for kind, eid, toks in prefix_entities_in_order(q):
            if (kind, eid) in ekv:
                continue
            n = len(toks)
            k = _rand((L, n, Hkv, d), 1.0, 1000 + len(ekv))
            v = _rand((L, n, Hkv, d), 1.0, 2000 + len(ekv))
            B.bat_kv_append(pool.handle, kind, eid, k, v, n)
            ekv[(kind, eid)] = (k.float().cpu().numpy(), v.float().cpu().numpy())
    QA = B.QueryArray(queries)
    plan = B.bat_plan_create(pool.handle, cfg["q_heads"] // cfg["kv_heads"], QA)
    S = [B.bat_plan_query_info(plan, b)["S"] for b in range(len(queries))]
    B.bat_plan_destroy(plan)
    M = sum(S)
    nqkv = (cfg["q_heads"] + 2 * Hkv) * d
    qkv = _rand((M, nqkv), 1.0, 77)
    out = torch.zeros(M, cfg["q_heads"] * d, dtype=torch.bfloat16, device="cuda")
    B.bat_debug_attention_layer(pool.handle, model.handle, QA, layer, qkv, out, True)
    torch.cuda.synchronize()
    qkv_np, out_np = qkv.float().cpu().numpy(), out.float().cpu().numpy()
    off = 0
    worst = -1.0
    for q, s in zip(queries, S):
        ref = oracle_attention_layer(cfg, q, ekv, qkv_np[off:off + s], layer)
        got = out_np[off:off + s].reshape(ref.shape)
        worst = max(worst, max_excess(got, ref))
        err = np.abs(got - ref)
        print(f"attention layer {cfg_name} {q.order} cache={q.use_cache}: max|err| {err.max():.4g} "
              f"mean|err| {err.mean():.3g} max|ref| {np.abs(ref).max():.3g} excess {worst:.4g}")
        off += s
    pool.close()
    model.close()
    return worst


@pytest.mark.parametrize("order", ["IP", "UP", "RE"])
def test_attention_layer_tiny(B, order):
    def qs(cfg):
        return [synth.make_query(0, cfg, 3, 16, [11, 22, 33, 44], (8, 8), 2,
                                 "UP" if order == "UP" else "IP", use_cache=(order != "RE"))]
    assert _attention_case(B, "tiny", qs) <= 0


@pytest.mark.parametrize("order", ["IP", "UP", "RE"])
def test_attention_layer_tiny_multi_tile_ragged(B, order):
    def qs(cfg):
        return [synth.make_query(1, cfg, 4, 150, list(range(100, 112)), (12, 20), 3,
                                 "UP" if order == "UP" else "IP", use_cache=(order != "RE"))]
    assert _attention_case(B, "tiny", qs) <= 0


@pytest.mark.parametrize("order", ["IP", "UP", "RE"])
def test_attention_layer_small_gqa6(B, order):
    def qs(cfg):
        return [synth.make_query(2, cfg, 5, 100, list(range(200, 220)), (16, 16), 8,
                                 "UP" if order == "UP" else "IP", use_cache=(order != "RE"))]
    assert _attention_case(B, "small", qs) <= 0


def test_attention_layer_mixed_batch_with_header(B):
    def qs(cfg):
        return [synth.make_query(3, cfg, 6, 40, list(range(300, 310)), (5, 17), 4, "IP", n_header=3),
                synth.make_query(3, cfg, 7, 90, list(range(300, 306)), (5, 17), 2, "UP"),
                synth.make_query(3, cfg, 8, 33, list(range(305, 312)), (5, 17), 1, "IP", use_cache=False)]
    assert _attention_case(B, "small", qs, layer=0) <= 0

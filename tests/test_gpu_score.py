"""The score kernel on its own, through bat_score's logits output:
z_i = W_out[v_i] . hf compared ELEMENTWISE with the fp64 oracle (oracle/score.py) on the
same fp32 hidden states and bf16 identifier rows, s = softmax(z) on a relative scale, and
the top-k exactly wherever the oracle's consecutive scores are separated by more than the
kernel's fp32 rounding.  N spans the paper's candidate counts (100-200), small and maximal sets,
ragged rows (n_items < n_max) and an empty row (n_items = 0: scores 0, top-k -1)."""
import numpy as np
import pytest

import synth
from oracle.score import score as oracle_score

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def B():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
    bat.lib()
    return bat


@pytest.fixture(scope="module")
def model(B):
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel
    cfg = synth.model_config("small")
    W = synth.Weights(cfg, seed=5)
    return cfg, W, DeviceModel(cfg, W)


@pytest.mark.parametrize("n_list", [[4], [20, 7, 1], [100, 100], [200, 150, 0, 199], [4096]])
def test_score_kernel_logits_scores_topk(B, model, n_list):
    cfg, W, m = model
    H, V = cfg["hidden"], cfg["vocab"]
    rng = np.random.default_rng(sum(n_list))
    Bn, n_max = len(n_list), max(max(n_list), 1)
    k = min(10, n_max)
    hf = rng.standard_normal((Bn, H)).astype(np.float32)
    labels = np.zeros((Bn, n_max), np.int32)
    for b, n in enumerate(n_list):
        labels[b, :n] = rng.integers(0, V, size=n)
    hidden = torch.tensor(hf, device="cuda")
    lab = torch.tensor(labels, device="cuda")
    nit = torch.tensor(n_list, dtype=torch.int32, device="cuda")
    scores = torch.full((Bn, n_max), 7.0, device="cuda")
    logits = torch.full((Bn, n_max), 7.0, device="cuda")
    topk = torch.full((Bn, k), 7, dtype=torch.int32, device="cuda")
    B.bat_score(m.handle, hidden, lab, nit, Bn, n_max, scores, k, topk, logits=logits)
    torch.cuda.synchronize()
    z_g, s_g, t_g = logits.double().cpu().numpy(), scores.double().cpu().numpy(), topk.cpu().numpy()
    for b, n in enumerate(n_list):
        assert np.all(z_g[b, n:] == 0) and np.all(s_g[b, n:] == 0)
        if n == 0:
            assert np.all(t_g[b] == -1)
            continue
        rows = np.asarray(W.lm_head_rows(labels[b, :n]), np.float64)
        z, s, top = oracle_score(rows, hf[b].astype(np.float64), min(k, n))
        # fp32 accumulation of H bf16 x fp32 products: |err| <~ H * 2^-24 * sum|w h|
        bound = 1e-5 * (np.abs(rows) @ np.abs(hf[b].astype(np.float64))) + 1e-6
        assert np.all(np.abs(z_g[b, :n] - z) <= bound), np.max(np.abs(z_g[b, :n] - z) - bound)
        np.testing.assert_allclose(np.log(s_g[b, :n]), np.log(s), rtol=0, atol=1e-4)
        assert abs(s_g[b, :n].sum() - 1.0) < 1e-5
        # top-k: exact where the oracle's consecutive scores differ by more than the fp32 noise
        srt = s[top]
        for r in range(min(k, n)):
            if r + 1 < len(srt) and srt[r] - srt[r + 1] <= 1e-4 * srt[r]:
                break
            assert t_g[b, r] == top[r], (b, r)
        assert np.all(t_g[b, n:] == -1) if n < k else True

"""Edge cases of the bipartite prefill on the GPU, each against the fp64 oracle (2e-2 abs/rel on
hf and s): no user tokens (IP: the suffix is the instruction alone), a single one-token item, items
of exactly one page and of one page + 1 token (16 / 17 tokens: page-boundary slots), a single
instruction token, one long request whose suffix spans many q-tiles with a ragged tail, and a
batch mixing all of them (different suffix lengths, q-tile counts and prefix sides)."""
import numpy as np
import pytest

import synth
from oracle import model as om
from tests.gpu_util import max_excess

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def env():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel
    cfg = synth.model_config("small")
    W = synth.Weights(cfg, seed=1)
    return bat, cfg, W, DeviceModel(cfg, W)


def _serve_check(env, qs):
    bat, cfg, W, model = env
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DevicePool, prefill_missing_entities
    pool = DevicePool(cfg, 2048)
    prefill_missing_entities(pool, model, qs)
    Bn, n_max = len(qs), max(q.n_items for q in qs)
    hidden = torch.empty(Bn, cfg["hidden"], device="cuda")
    bat.bat_bipartite_prefill(pool.handle, model.handle, bat.QueryArray(qs), hidden)
    labels = np.zeros((Bn, n_max), np.int32)
    for b, q in enumerate(qs):
        labels[b, : q.n_items] = q.labels
    scores = torch.empty(Bn, n_max, device="cuda")
    bat.bat_score(model.handle, hidden, torch.tensor(labels, device="cuda"),
                  torch.tensor([q.n_items for q in qs], dtype=torch.int32, device="cuda"), Bn, n_max, scores)
    torch.cuda.synchronize()
    hf, s = hidden.double().cpu().numpy(), scores.double().cpu().numpy()
    worst = -1.0
    for b, q in enumerate(qs):
        ref = om.run_query(cfg, W, q, "full")
        worst = max(worst, max_excess(hf[b], ref["hf"]), max_excess(s[b, : q.n_items], ref["s"]))
    pool.close()
    assert worst <= 0, worst
    return worst


def test_ip_without_user_tokens(env):
    cfg = env[1]
    _serve_check(env, [synth.make_query(2, cfg, 1, 0, list(range(10, 18)), (16, 16), 3, "IP")])


def test_single_one_token_item_and_single_instruction_token(env):
    cfg = env[1]
    qs = [synth.make_query(2, cfg, 2, 40, [77], (1, 1), 1, o) for o in ("IP", "UP")]
    _serve_check(env, qs)


@pytest.mark.parametrize("item_len", [16, 17])
def test_page_boundary_item_lengths(env, item_len):
    cfg = env[1]
    qs = [synth.make_query(3, cfg, 3, 33, list(range(20, 32)), (item_len, item_len), 4, o) for o in ("IP", "UP")]
    _serve_check(env, qs)


def test_long_suffix_many_q_tiles_ragged_tail(env):
    """|U| = 700 in IP: 706 suffix tokens = 34 q-tiles of 21 tokens (GQA 6) with a ragged last one."""
    cfg = env[1]
    _serve_check(env, [synth.make_query(4, cfg, 4, 700, list(range(40, 60)), (9, 23), 6, "IP")])


def test_mixed_edge_batch(env):
    cfg = env[1]
    qs = [synth.make_query(5, cfg, 5, 0, [1, 2, 3], (16, 16), 1, "IP"),
          synth.make_query(5, cfg, 6, 300, [4], (17, 17), 2, "UP"),
          synth.make_query(5, cfg, 7, 129, list(range(5, 25)), (1, 16), 8, "IP"),
          synth.make_query(5, cfg, 8, 64, list(range(25, 30)), (16, 16), 3, "UP", use_cache=False)]
    _serve_check(env, qs)

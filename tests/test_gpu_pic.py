"""GPU parity of the selective-recompute variant of Item-as-prefix (PAPER.md
P:265 / P:476, reading DESIGN.md R25): every item's last k tokens recomputed after U, the heads
served from the same cached item entries.  No new kernel: the planner expresses PIC as trimmed
prefix page lists + extra suffix tokens (segment = item, positions after U), so the production
bf16 path and the fp32 mode run it unchanged.  Checked against the oracle's full recompute of the
PIC prompt at 2e-2 (bf16: hf, the kernel's logits z, s) and 1e-5 (fp32 mode), in batches mixing
PIC, plain IP, UP and RE requests; plus the layer-level attention of a PIC batch."""
import numpy as np
import pytest

import synth
from tests import test_gpu_fp32 as F
from tests import test_gpu_kernels as K
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


def _pic_batch(cfg, seed=0):
    qs = []
    for i, (n_u, order, k, cache) in enumerate([(40, "IP", 1, True), (90, "IP", 4, True), (25, "IP", 100, True),
                                                 (60, "IP", 0, True), (130, "UP", 0, True), (33, "IP", 3, False)]):
        # the header request gets its own items: an item's cached KV is computed in its request's
        # context (after the header, reading R3), so it cannot be shared with header-less requests
        ids = list(range(300, 312)) if i == 1 else list(range(70 + 2 * i, 82 + 2 * i))
        q = synth.make_query(seed, cfg, 20 + i, n_u, ids, (5, 19), 1 + i % 3,
                             order, use_cache=cache, n_header=(3 if i == 1 else 0))
        q.pic_tail = k
        qs.append(q)
    return qs


@pytest.mark.parametrize("cfg_name", ["tiny", "small"])
def test_pic_bf16_parity(B, cfg_name):
    qs = _pic_batch(synth.model_config(cfg_name))
    cfg, W, out = G._run(B, cfg_name, qs)
    G._check(cfg, W, qs, out)


def test_pic_fp32_parity(B):
    F._run_check(B, "small", _pic_batch(synth.model_config("small"), seed=2))


def test_pic_attention_layer(B):
    def qs(cfg):
        return _pic_batch(cfg, seed=4)
    assert K._attention_case(B, "small", qs, layer=1) <= 0

"""The opt-in attention kernels (BAT_ATTN=pair: CTA-pair cta_group::2 with double-buffered S;
BAT_ATTN=db: 1-CTA with 64-key double-buffered S) against the same fp64 references as the
default kernel: the layer-level attention tests (O within 2e-2 abs/rel of the oracle's masked
attention) and the end-to-end small-model parity tests.  The kernel is chosen once per process
(environment), so each variant runs in a child pytest."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("variant", ["pair", "db"])
def test_attention_variant_parity(variant):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    env = dict(os.environ, BAT_ATTN=variant)
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
                        "tests/test_gpu_kernels.py", "-k", "attention",
                        "tests/test_gpu_parity.py"], cwd=ROOT, env=env, capture_output=True, text=True,
                       timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
    assert " passed" in r.stdout

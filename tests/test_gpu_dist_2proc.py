"""Two processes, one GPU: the multi-process serving path of bench.py --gpus N end to end on real
hardware (tests/_dist2_worker.py): Alg. 1 placement over world = 2, CUDA-IPC arena export /
attach, page-table all_gather, cold-item pulls from the peer process's arena, and serving —
every rank's results must match the fp64 oracle (2e-2 abs/rel on hf)."""
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_two_process_cold_item_pull_and_serving(tmp_path):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    port = _free_port()
    outs = [str(tmp_path / f"r{r}.txt") for r in range(2)]
    procs = [subprocess.Popen([sys.executable, os.path.join(ROOT, "tests", "_dist2_worker.py"), str(r), "2", str(port),
                               outs[r]], cwd=ROOT, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)
             for r in range(2)]
    logs = [p.communicate(timeout=600)[0] for p in procs]
    for p, log in zip(procs, logs):
        assert p.returncode == 0, log[-3000:]
    total_local = 0
    for o in outs:
        rank, n_local, n_remote, n_cold, pulled, worst = open(o).read().split()
        total_local += int(n_local)
        assert int(n_remote) > 0 and int(pulled) == int(n_cold) > 0  # the peer's items were pulled
        assert float(worst) <= 0, (rank, worst)
    assert total_local >= 48  # every item stored somewhere (replicated ones on both)


def test_bench_two_ranks_on_one_gpu_prints_a_valid_line():
    """bench.py's N > 1 path (torchrun, in-run calibration of Alg. 1's B and t, HRCS placement, IPC
    exchange, request routing, staged cold pulls one batch ahead inside the timed region,
    max-over-ranks timing) end to end with two ranks sharing the GPU (BAT_BENCH_SHARED_GPU=1: gloo
    bootstrap).  Only the contract is checked — two ranks on one GPU time nothing real."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import json
    env = dict(os.environ, BAT_BENCH_SHARED_GPU="1")
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), "bench.py", "--gpus", "2",
                        "--steps", "2", "--warmup", "1", "--batch", "4", "--corpus", "512", "--no-cpu-baseline"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1  # rank 0 only
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["config"]["global_batch"] == 8 and d["value"] > 0
    h = d["config"]["hrcs"]
    assert h["cold_pages_pulled_per_step"] > 0 and d["e2e"]["value"] > 0
    assert h["pull_gbs"] > 0 and h["t_request_s"] > 0  # Alg. 1 inputs measured in-run

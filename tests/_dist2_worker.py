"""Worker of tests/test_gpu_dist_2proc.py: one rank of a 2-process data-parallel serving round on
ONE GPU (both ranks on cuda:0, gloo bootstrap).  Exercises the real multi-process path of
bench.py --gpus N: Alg. 1 placement, CUDA-IPC export/attach of the pool arenas, all_gather of the
owners' page tables, cold-item pulls from the peer's arena (bat_kv_fetch), serving."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch
import torch.distributed as dist

import synth
from oracle import model as om
from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
from paper_conf_asplos_0017wzlxszh0w26_b200 import dist as bdist
from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel, DevicePool, prefill_missing_entities


def main(rank: int, world: int, port: int, out: str):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    cfg = synth.model_config("tiny")
    W = synth.Weights(cfg, seed=1)
    model = DeviceModel(cfg, W)
    pool = DevicePool(cfg, 1024, rank=rank, world=world)
    corpus = 48
    freq = synth.zipf_weights(corpus)
    r, owner = bdist.place_items(freq, 0.2, world)
    mine = bdist.local_items(owner, rank)
    toks = [synth.item_tokens(1, i, synth.item_length(i, 8, 8, 1), cfg["vocab"]) for i in mine]
    bat.bat_kv_prefill_entities(pool.handle, model.handle, bat.BAT_ENT_ITEM, mine, toks, 0)
    n_remote = bdist.exchange_remote(pool.handle, owner, rank, world)
    rng = np.random.default_rng(100 + rank)
    qs = [synth.make_query(1, cfg, 10 * rank + b, 16 + 4 * b, synth.distinct_label_items(1, cfg, 6, rng, corpus),
                           (8, 8), 2, "IP") for b in range(3)]
    cold = bdist.cold_items(qs, owner, rank)
    pulled = bdist.fetch_cold(pool.handle, cold)
    prefill_missing_entities(pool, model, qs)  # nothing left to compute: every item is local now
    hidden = torch.empty(len(qs), cfg["hidden"], device="cuda")
    bat.bat_bipartite_prefill(pool.handle, model.handle, bat.QueryArray(qs), hidden)
    torch.cuda.synchronize()
    worst = -1.0
    hf = hidden.double().cpu().numpy()
    for b, q in enumerate(qs):
        ref = om.run_query(cfg, W, q, "full")
        worst = max(worst, float(np.max(np.abs(hf[b] - ref["hf"]) - (2e-2 + 2e-2 * np.abs(ref["hf"])))))
    dist.barrier()
    with open(out, "w") as f:
        f.write(f"{rank} {len(mine)} {n_remote} {len(cold)} {pulled} {worst}\n")
    pool.close()
    model.close()
    dist.destroy_process_group()


if __name__ == "__main__":
    main(int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4])

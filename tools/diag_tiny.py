"""Diagnostic: tiny end-to-end hidden state vs the oracle, per element."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
from oracle import model as om
from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel, DevicePool, prefill_missing_entities
cfg = synth.model_config("tiny"); W = synth.Weights(cfg, seed=1)
model = DeviceModel(cfg, W)
for order, uc in (("IP", True), ("IP", False), ("UP", True)):
    q = synth.make_query(0, cfg, 3, 16, [11, 22, 33, 44], (8, 8), 2, order, use_cache=uc)
    pool = DevicePool(cfg, 256)
    prefill_missing_entities(pool, model, [q])
    h = torch.empty(1, cfg["hidden"], device="cuda")
    bat.bat_bipartite_prefill(pool.handle, model.handle, bat.QueryArray([q]), h)
    torch.cuda.synchronize()
    got = h[0].double().cpu().numpy()
    ref = om.run_query(cfg, W, q, "full")["hf"]
    err = np.abs(got - ref)
    i = int(np.argmax(err - (0.02 + 0.02 * np.abs(ref))))
    print(order, uc, "max|err|", err.max().round(5), "worst elem", i, got[i].round(5), ref[i].round(5))
    np.save(f"gpurun_out/hf_{order}_{uc}_{os.environ.get('PP','x')}.npy", got)
    pool.close()

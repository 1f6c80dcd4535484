"""Mask-sensitivity guard at full size (R12): the fp64 oracle with a plain causal mask
(items see each other) must move the identifier logits z of a configs[1] request by > 10 x atol
at the full-size parity init, or the parity tests could not see a mask bug.
usage: python tools/mask_guard_full.py [mlp_std] [order] [model] [layers] [n_user] [n_items] [seed]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, synth
from oracle import model as om
from oracle.sequence import causal_mask
cfg = synth.model_config(sys.argv[3] if len(sys.argv) > 3 else "qwen2-1.5b")
if len(sys.argv) > 4: cfg["layers"] = int(sys.argv[4])
cfg["mlp_std"] = float(sys.argv[1]) if len(sys.argv) > 1 else 0.01
order = sys.argv[2] if len(sys.argv) > 2 else "IP"
W = synth.Weights(cfg, seed=int(sys.argv[7]) if len(sys.argv) > 7 else 1)
n_user = int(sys.argv[5]) if len(sys.argv) > 5 else 512
n_items = int(sys.argv[6]) if len(sys.argv) > 6 else 100
rng = np.random.default_rng(7)
q = synth.make_query(0, cfg, 1000, n_user, synth.distinct_label_items(0, cfg, n_items, rng, 8192, synth.zipf_weights(8192)),
                     (16, 16), 8, order)
good = om.run_query(cfg, W, q, "full")
bad = om.run_query(cfg, W, q, "full", mask_fn=lambda seg: causal_mask(len(seg)))
print(f"mlp_std {cfg['mlp_std']} {order}: max|dz| wrong mask {np.abs(good['z'] - bad['z']).max():.3f} "
      f"(guard > {10 * 2e-2}); z std {good['z'].std():.3f}; max s {good['s'].max():.3f}")

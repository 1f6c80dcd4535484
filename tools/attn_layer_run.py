"""One Qwen2-1.5B-shaped attention layer (configs[1] IP batch, random KV) through
bat_debug_attention_layer, a few times — the command ncu profiles (tools/gpu/run_ncu_attn.sh)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DevicePool, DeviceModel
from bench import device_weights
cfg = synth.model_config("qwen2-1.5b"); cfg["layers"] = 2
B = int(os.environ.get("B", "64")); order = os.environ.get("ORDER", "IP")
dev = torch.device("cuda", 0)
model = DeviceModel(cfg, tensors=device_weights(cfg, 1, dev))
pool = DevicePool(cfg, 20000)
rng = np.random.default_rng(0)
qs = [synth.make_query(0, cfg, 1000 + b, 512, rng.choice(4000, 100, replace=False), (16, 16), 8, order) for b in range(B)]
L, Hkv, d = cfg["layers"], cfg["kv_heads"], cfg["head_dim"]
seen = set()
for q in qs:
    ents = [(bat.BAT_ENT_USER, q.user_id, len(q.user_tok))] if order == "UP" else [(bat.BAT_ENT_ITEM, int(i), 16) for i in q.item_ids]
    for kind, eid, n in ents:
        if (kind, eid) in seen: continue
        seen.add((kind, eid))
        k = torch.randn(L, n, Hkv, d, device=dev).to(torch.bfloat16); v = torch.randn_like(k)
        bat.bat_kv_append(pool.handle, kind, eid, k, v, n)
QA = bat.QueryArray(qs)
plan = bat.bat_plan_create(pool.handle, 6, QA)
M = sum(bat.bat_plan_query_info(plan, b)["S"] for b in range(B))
bat.bat_plan_destroy(plan)
qkv = torch.randn(M, 2048, device=dev).to(torch.bfloat16)
out = torch.empty(M, 1536, device=dev, dtype=torch.bfloat16)
for _ in range(int(os.environ.get("REPS", "3"))):
    bat.bat_debug_attention_layer(pool.handle, model.handle, QA, 1, qkv, out)
torch.cuda.synchronize()
print("done")

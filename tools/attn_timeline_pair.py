"""Run one Qwen2-1.5B-shaped attention layer (configs[1] IP batch, random KV) through
bat_debug_attention_layer, time it, and print CTA 0's clock64 timeline (BAT_ATTN_TIMELINE)
of the double-buffered kernel (per 64-key sub-tile)."""
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
info = [bat.bat_plan_query_info(plan, b) for b in range(B)]
bat.bat_plan_destroy(plan)
M = sum(i["S"] for i in info); live = sum(i["n_live_pairs"] for i in info)
qkv = torch.randn(M, 2048, device=dev).to(torch.bfloat16)
out = torch.empty(M, 1536, device=dev, dtype=torch.bfloat16)
for _ in range(3): bat.bat_debug_attention_layer(pool.handle, model.handle, QA, 1, qkv, out)
torch.cuda.synchronize()
os.environ["BAT_ATTN_TIMELINE"] = "gpurun_out/attn_timeline.txt"
bat.bat_profile_enable(model.handle, True)
bat.bat_debug_attention_layer(pool.handle, model.handle, QA, 1, qkv, out)
del os.environ["BAT_ATTN_TIMELINE"]
# timing (stage + attention) with events
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10): bat.bat_debug_attention_layer(pool.handle, model.handle, QA, 1, qkv, out)
e1.record(); torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 10
print(f"{order} B={B}: stage+attention {ms:.3f} ms/layer (host sync included); flops {4*128*12*live/1e9:.1f} GF -> {4*128*12*live/ms/1e9:.0f} TFLOP/s lower bound")
t = np.loadtxt("gpurun_out/attn_timeline.txt").astype(np.int64)
names = ["S_iss", "mma_wP", "mma_P", "mma_V", "PV_iss", "sm_wS", "sm_S", "sm_max", "sm_dec", "sm_done", "ld_K", "ld_V", "S_kok", "sm_arr", "sm_top"]
t0 = t[t > 0].min()
print("tile " + " ".join(f"{nm:>8}" for nm in names))
for x in range(64):
    if t[4, x] == 0:
        break
    print(f"{x:4d} " + " ".join(f"{(t[e, x] - t0) if t[e, x] else -1:8d}" for e in range(15)))
ok = (t[6] > 0) & (t[9] > 0)
print("softmax per tile: S wait %.0f, ld+max %.0f, decision wait %.0f, rest %.0f" % (
    np.mean((t[6]-t[5])[ok]), np.mean((t[7]-t[6])[ok]), np.mean((t[8]-t[7])[ok]), np.mean((t[9]-t[8])[ok])))
pv = t[4][t[4] > 0]
print("PV interval (clk per tile) median %.0f" % np.median(np.diff(pv)))
ok2 = (t[1] > 0) & (t[2] > 0)
print("MMA: P wait %.0f, V wait %.0f, PV issue %.0f" % (np.mean((t[2]-t[1])[ok2]), np.mean((t[3]-t[2])[ok2]), np.mean((t[4]-t[3])[ok2])))

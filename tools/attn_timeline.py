"""Run one Qwen2-1.5B-shaped attention layer (configs[1] IP batch, random KV) through
bat_debug_attention_layer, time it, and print CTA 0's clock64 timeline (BAT_ATTN_TIMELINE)."""
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
NU = int(os.environ.get("NU", "512")); NI = int(os.environ.get("NI", "100"))
qs = [synth.make_query(0, cfg, 1000 + b, NU, rng.choice(4000, NI, replace=False), (16, 16), 8, order) for b in range(B)]
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
names = ["ld_kwait", "ld_kgot", "ld_kiss", "ld_vbwait", "ld_vbgot", "mma_top", "mma_p0", "mma_vful",
         "mma_pvdone", "mma_Skful", "mma_end", "sm0_s", "sm0_fast", "sm0_p", "sm1_s", "sm1_p",
         "sm0_16", "sm0_17", "sm0_max", "sm0_pst"]
if os.environ.get("H64"):  # the h64 kernel's events (per 64-key half tile)
    names = ["vfull0", "pv0iss", "s0_kwait", "s0_kgot", "-", "mma_top", "mma_p0", "mma_p1", "mma_s0", "-", "mma_end", "t0_s", "-",
             "t0_p", "t1_s", "t1_p", "-", "-", "t0_dec", "t0_refok"]
t0 = t[t > 0].min()
n = int(max((t[e] > 0).sum() for e in range(t.shape[0])))
print("tile " + " ".join(f"{nm:>10}" for nm in names))
for x in range(min(n, 64)):
    print(f"{x:4d} " + " ".join(f"{(t[e, x] - t0) if t[e, x] else -1:10d}" for e in range(20)))

# ---- per-work-item records (BAT_ATTN_ITEMS): where the time per item goes, per CTA
os.environ["BAT_ATTN_ITEMS"] = "gpurun_out/attn_items.txt"
bat.bat_debug_attention_layer(pool.handle, model.handle, QA, 1, qkv, out)
del os.environ["BAT_ATTN_ITEMS"]
it = np.loadtxt("gpurun_out/attn_items.txt").astype(np.int64)  # t_q t_s0 t_lastpv t_end kt_n cta
cta = it[:, 5]
print(f"work items {len(it)}  k-tiles mean {it[:,4].mean():.2f} min {it[:,4].min()} max {it[:,4].max()}")
tot_span, tot_busy = [], []
per_tile, gaps, epi, head = [], [], [], []
for c in np.unique(cta):
    r = it[cta == c]
    r = r[np.argsort(r[:, 0])]
    tot_span.append(r[-1, 3] - r[0, 0])
    per_tile += list((r[:, 2] - r[:, 1]) / np.maximum(1, r[:, 4] - 1))
    epi += list(r[:, 3] - r[:, 2])
    head += list(r[:, 1] - r[:, 0])
    gaps += list(r[1:, 0] - r[:-1, 2])
span = np.array(tot_span)
print(f"CTA span (clk): mean {span.mean():.0f} min {span.min()} max {span.max()}  items/CTA {len(it)/len(span):.2f}")
print(f"per item: q->S0 issued {np.mean(head):.0f}  S0..lastPV per k-tile {np.mean(per_tile):.0f}  "
      f"lastPV->epilogue done {np.mean(epi):.0f}  lastPV(i)->q_full(i+1) {np.mean(gaps):.0f}")

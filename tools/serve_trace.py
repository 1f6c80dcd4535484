"""Serving study on one B200 (the analog of PAPER.md Fig. 5 / Fig. 6 on a
synthetic trace — the real traces are out of scope): Qwen2-1.5B-shaped random-weight model,
requests from synth.request_trace (Zipf user activity, lognormal profile lengths), 100 candidate
items of 16 tokens drawn Zipf(1.093) from a precomputed item corpus, a user-prefix cache of
--user-cache-frac of all distinct users' pages.  For each policy (RE, UP, IP, greedy P:366,
hotness-aware BAT P:377) the whole trace is served through runtime.TraceServer (scheduler +
cache actions + bat_bipartite_prefill + bat_score) and timed end to end on the wall clock
(host scheduling and user-prefix computation included).  Prints one JSON line per policy:
requests/s, P:441 hit rate (reused prefix tokens / prompt tokens), speedups vs RE / UP."""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
from bench import device_weights
from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel, DevicePool, TraceServer, prefill_missing_entities

ap = argparse.ArgumentParser()
ap.add_argument("--requests", type=int, default=600)
ap.add_argument("--users", type=int, default=300)
ap.add_argument("--corpus", type=int, default=4096)
ap.add_argument("--user-cache-frac", type=float, default=0.2)
ap.add_argument("--window", type=float, default=20.0)
ap.add_argument("--batch", type=int, default=32)
ap.add_argument("--policies", default="re,up,ip,greedy,hotness")
args = ap.parse_args()

cfg = synth.model_config("qwen2-1.5b")
dev = torch.device("cuda", 0)
model = DeviceModel(cfg, tensors=device_weights(cfg, 1, dev))
trace = synth.request_trace(11, args.requests, args.users, rate=20.0, tau_i=1600)
rng = np.random.default_rng(3)
zp = synth.zipf_weights(args.corpus)
items = [synth.distinct_label_items(0, cfg, 100, rng, args.corpus, zp) for _ in trace]
reqs = [(t, u, tu, it) for (t, u, tu, _), it in zip(trace, items)]
distinct_pages = sum(-(-tu // 16) for tu in {u: tu for _, u, tu, _ in trace}.values())
cap = int(args.user_cache_frac * distinct_pages)
res = {}
for pol in args.policies.split(","):
    pool = DevicePool(cfg, args.corpus + cap + 4096)
    # the item corpus is resident before serving (offline item precompute)
    warm = [synth.make_query(0, cfg, 10 ** 6, 8, synth.distinct_label_items(0, cfg, 100, rng, args.corpus, zp),
                             (16, 16), 8, "IP")]
    all_items = np.arange(args.corpus)
    for s in range(0, args.corpus, 512):
        q = synth.make_query(0, cfg, 10 ** 6, 8, all_items[s:s + 512], (16, 16), 8, "IP")
        prefill_missing_entities(pool, model, [q])
    torch.cuda.synchronize()
    srv = TraceServer(pool, model, pol, cap, args.window, seed=0)
    t0 = time.perf_counter()
    srv.serve(reqs, batch=args.batch)
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    st = srv.stats()
    res[pol] = dict(policy=pol, requests_per_s=len(reqs) / dt, seconds=dt, hit_rate=st["reused"] / st["tokens"],
                    up=st["up"], ip=st["ip"], user_hits=st["hits"], user_cache_pages=cap)
    srv.close()
    pool.close()
    print(json.dumps(res[pol]), flush=True)
if "re" in res:
    for pol, r in res.items():
        r["speedup_vs_re"] = r["requests_per_s"] / res["re"]["requests_per_s"]
        if "up" in res:
            r["speedup_vs_up"] = r["requests_per_s"] / res["up"]["requests_per_s"]
print(json.dumps({"summary": res, "trace": dict(requests=args.requests, users=args.users, corpus=args.corpus,
                                                user_cache_frac=args.user_cache_frac, window=args.window)}))

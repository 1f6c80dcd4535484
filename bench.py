#!/usr/bin/env python
"""bench.py — throughput of the BAT bipartite prefill on B200 (one JSON line on rank 0).

Workload (BASELINE.json configs[1]): Qwen2-1.5B-shaped GR ranking model (28 layers, hidden
1536, 12 Q / 2 KV heads, d 128, ffn 8960, vocab 151936; random bf16 weights), requests of
1 user of 512 tokens + 100 candidate items of 16 tokens + 8 instruction tokens, served
Item-as-prefix (the prefix side P:366's larger-side rule picks for |U| = 512 < 1600
item tokens): the 100 items' KV is read from the paged pool, the 520 user + instruction
tokens are computed through the 28 layers, then the 100 items are scored.
A step = one batch of --batch requests (all §8(a) rows: plan, embed, 28 x [norm, QKV,
RoPE/stage, bipartite attention, O, norm, SwiGLU MLP], last-layer trim, final norm, score).
Items are drawn Zipf(1.093) from a corpus whose KV was precomputed with the same model
(bat_kv_prefill_entities, the prefix-miss path) before timing.

value  = requests/s with inputs resident in HBM (pre-built device plans, bat_prefill_plan).
e2e    = requests/s through the public call with HOST inputs (bat_bipartite_prefill plans and
         uploads every step; labels H2D from pinned memory; scores + top-k D2H every step).
N > 1  = one process per GPU (torchrun); every rank serves its own batches (weak scaling);
         items are placed hot-replicated / cold-sharded by Algorithm 1 and every
         rank pulls the cold items it needs from their owners' pools over NVLink (CUDA IPC
         mapped arenas, bat_kv_fetch) inside the timed region.

--impl reference times the fp64 CPU oracle (oracle/, full recompute, the plain definition)
on the host cores on a bounded sample (one layer of one request per step, x28 layers).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import synth  # noqa: E402

METRIC = "ranking queries/sec & prefill tokens/sec per B200 at 1/2/4/8 GPUs; % tensor peak"
WORKLOAD = ("configs[1]: Qwen2-1.5B-shaped (28 layers, hidden 1536, 12 Q / 2 KV heads, d=128), "
            "1 user of 512 tokens + 100 items of 16 tokens, bf16, item-as-prefix")


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="bat", choices=["bat", "reference"])
    ap.add_argument("--batch", type=int, default=64, help="requests per step per GPU")
    ap.add_argument("--model", default="qwen2-1.5b", choices=["qwen2-1.5b", "qwen2-7b", "llama3-1b"],
                    help="model shape (the driver's line is qwen2-1.5b = configs[1])")
    ap.add_argument("--n-user", type=int, default=512)
    ap.add_argument("--n-items", type=int, default=100)
    ap.add_argument("--item-len", type=int, default=16)
    ap.add_argument("--n-instr", type=int, default=8)
    ap.add_argument("--corpus", type=int, default=8192, help="items in the corpus")
    ap.add_argument("--plans", type=int, default=4, help="distinct pre-built batches cycled")
    ap.add_argument("--alpha", type=float, default=0.1, help="Alg. 1 communication/compute ratio")
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=20.0, help="seconds of oracle time")
    return ap.parse_args()


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return dict(hbm=d["hbm_gbs"], bf16=d["bf16_tflops"], bf16_sus=d.get("bf16_tflops_sustained", d["bf16_tflops"]),
                    src="measured (MEASURED_PEAKS.json)")
    return dict(hbm=6650.0, bf16=1590.0, bf16_sus=1400.0, src="fallback (B200_PROFILING.md)")


# ------------------------------------------------------------------------- clocks
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return dict(sm_mhz=None, sm_max_mhz=None, reasons=["nvidia-smi unavailable"])
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 8:
                continue
            try:
                sm.append(float(parts[0]))
                mx = float(parts[1])
            except ValueError:
                continue
            for n, v in zip(names, parts[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return dict(sm_mhz=statistics.median(sm) if sm else None, sm_max_mhz=mx,
                    reasons=sorted(reasons), samples=len(sm))


# ---------------------------------------------------------------------- weights
def device_weights(cfg, seed, device):
    """Random-init bf16 weights of the architecture on the GPU (values do not affect timing;
    N(0, 0.02) matrices and biases, RMSNorm gains 1 + N(0, 0.1), tied lm_head)."""
    import torch
    g = torch.Generator(device=device).manual_seed(seed)
    bf = torch.bfloat16
    H, F, d, Hq, Hkv, V = cfg["hidden"], cfg["ffn"], cfg["head_dim"], cfg["q_heads"], cfg["kv_heads"], cfg["vocab"]
    rn = lambda *s, std=0.02, mean=0.0: (torch.randn(*s, generator=g, device=device) * std + mean).to(bf)
    embed = rn(V, H)
    layers = []
    for _ in range(cfg["layers"]):
        layers.append(dict(ln1=rn(H, std=0.1, mean=1.0), wqkv=rn((Hq + 2 * Hkv) * d, H), bqkv=rn((Hq + 2 * Hkv) * d),
                           wo=rn(H, Hq * d), ln2=rn(H, std=0.1, mean=1.0), wgu=rn(2 * F, H), wd=rn(H, F)))
    return dict(embed=embed, lm_head=embed if cfg["tied"] else rn(V, H), final_norm=rn(H, std=0.1, mean=1.0),
                layers=layers)


def make_queries(args, cfg, rng, user0, n, zipf_p):
    qs = []
    for b in range(n):
        items = synth.distinct_label_items(args.seed, cfg, args.n_items, rng, args.corpus, zipf_p)
        qs.append(synth.make_query(args.seed, cfg, user0 + b, args.n_user, items,
                                   (args.item_len, args.item_len), args.n_instr, "IP"))
    return qs


def algorithmic_flops_per_request(cfg, S, live_pairs, live_last):
    """Method FLOPs: linear layers on the S suffix rows at every layer except the last, whose
    O/MLP run only on the discriminant row (a8); attention 4*d*Hq per visible pair."""
    H, F, d, Hq, Hkv, L = cfg["hidden"], cfg["ffn"], cfg["head_dim"], cfg["q_heads"], cfg["kv_heads"], cfg["layers"]
    qkv = 2 * H * (Hq + 2 * Hkv) * d
    rest = 2 * (Hq * d) * H + 2 * H * 2 * F + 2 * F * H
    lin = S * (qkv + rest) * (L - 1) + S * qkv + 1 * rest
    attn = 4 * d * Hq * (live_pairs * (L - 1) + live_last)
    return lin + attn, lin, attn


# --------------------------------------------------------------------- oracle arm
def oracle_time_per_request(args, budget_s, max_layers=None):
    """Time the fp64 oracle (full recompute, explicit mask) on one configs[1] request,
    layer by layer until `budget_s`; returns (seconds per request extrapolated to L layers,
    sample description, threads)."""
    from oracle import model as om
    from oracle.sequence import bipartite_mask, build_sequence
    cfg = synth.model_config(args.model)
    W = synth.Weights(cfg, seed=args.seed)
    q = synth.make_query(args.seed, cfg, 0, args.n_user, list(range(args.n_items)),
                         (args.item_len, args.item_len), args.n_instr, "IP")
    toks, seg, pos = build_sequence(q.order, q.user_tok, q.item_toks, q.instr_tok)
    mask = bipartite_mask(seg)
    h = np.asarray(W.embed_rows(toks), np.float64)
    times = []
    L = cfg["layers"]
    for l in range(L if max_layers is None else min(L, max_layers)):
        w = W.layer(l)  # generation outside the timed region
        t0 = time.perf_counter()
        h, _, _ = om.layer_forward(cfg, w, h, pos, None, None, mask)
        times.append(time.perf_counter() - t0)
        if sum(times) >= budget_s:
            break
    per_layer = statistics.mean(times)
    threads = _blas_threads()
    sample = (f"1 request (T={len(toks)} tokens, full recompute as the oracle defines it), "
              f"{len(times)} of {L} layers timed, x{L} extrapolated")
    return per_layer * L, sample, threads, times


def _blas_threads():
    try:
        from threadpoolctl import threadpool_info
        n = [i.get("num_threads", 0) for i in threadpool_info() if i.get("user_api") == "blas"]
        return max(n) if n else len(os.sched_getaffinity(0))
    except Exception:
        return len(os.sched_getaffinity(0))


def run_reference(args):
    cfg = synth.model_config(args.model)
    S = args.n_user + args.n_instr
    from oracle import model as om
    from oracle.sequence import bipartite_mask, build_sequence
    W = synth.Weights(cfg, seed=args.seed)
    q = synth.make_query(args.seed, cfg, 0, args.n_user, list(range(args.n_items)),
                         (args.item_len, args.item_len), args.n_instr, "IP")
    toks, seg, pos = build_sequence(q.order, q.user_tok, q.item_toks, q.instr_tok)
    mask = bipartite_mask(seg)
    h0 = np.asarray(W.embed_rows(toks), np.float64)
    w = W.layer(0)
    times = []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        om.layer_forward(cfg, w, h0, pos, None, None, mask)
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
    t_req = statistics.mean(times) * cfg["layers"]
    value = 1.0 / t_req
    cores = _blas_threads()
    sample = (f"each step = 1 of 28 layers of 1 configs[1] request (T={len(toks)}, fp64 full recompute "
              f"with explicit mask), requests/s = 1 / (28 x mean layer time)")
    line = dict(metric=METRIC, value=value, unit="requests/s", n_gpus=args.gpus, steps=args.steps,
                warmup=args.warmup, ms_per_step=1e3 * statistics.mean(times), higher_is_better=True,
                scaling="weak", vs_baseline=None, dtype="f64", data="synthetic", impl="reference",
                config=dict(workload=WORKLOAD, batch=1, prefix="IP (oracle: full recompute)"),
                cpu_baseline=dict(value=value, unit="requests/s", cores=cores, kind="oracle", sample=sample),
                e2e=dict(value=value, unit="requests/s", h2d_bytes_per_step=0, d2h_bytes_per_step=0),
                prefill_tokens_per_s=value * (len(toks)))
    print(json.dumps(line))


# ------------------------------------------------------------------------ GPU arm
def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        if rank != 0:
            return
        run_reference(args)
        return

    import torch
    import torch.distributed as dist
    from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
    from paper_conf_asplos_0017wzlxszh0w26_b200.runtime import DeviceModel, DevicePool

    # BAT_BENCH_SHARED_GPU=1 (validation only): several ranks share the visible GPUs, bootstrap
    # and the max-over-ranks reduction go over gloo — exercises the N>1 code path on one GPU
    shared = os.environ.get("BAT_BENCH_SHARED_GPU") == "1"
    local = local % max(1, torch.cuda.device_count()) if shared else local
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    red_dev = torch.device("cpu") if shared else dev
    if world > 1:
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    cfg = synth.model_config(args.model)
    pk = peaks()

    # ---- model + pool
    model = DeviceModel(cfg, tensors=device_weights(cfg, 1234, dev), device=local)
    page_bytes = 16 * 2 * cfg["kv_heads"] * cfg["head_dim"] * cfg["layers"] * 2
    per_item_pages = (args.item_len + 15) // 16
    pages = args.corpus * per_item_pages * (2 if world > 1 else 1) + 1024
    pool = DevicePool(cfg, pages, device=local, rank=rank, world=world)
    stream = torch.cuda.current_stream(dev)

    # ---- item corpus: Zipf hotness, HRCS placement (Alg. 1) for N > 1
    from paper_conf_asplos_0017wzlxszh0w26_b200 import dist as bdist
    zipf_p = synth.zipf_weights(args.corpus)
    t_req_est = 0.0015  # s per request (prefill time t of Alg. 1 line 4, measured order on B200)
    owner = np.full(args.corpus, -1, np.int32)
    r_rep = 1.0
    r_max = None
    if world > 1:
        kv_tok = 2 * cfg["kv_heads"] * cfg["head_dim"] * cfg["layers"] * 2
        r_max = bdist.rmax_for_nvlink(770.0, t_req_est, args.alpha, args.n_items, args.item_len, world, kv_tok)
        r_rep, owner = bdist.place_items(zipf_p, r_max, world)
    local_items = bdist.local_items(owner, rank)
    item_toks = {i: synth.item_tokens(args.seed, i, args.item_len, cfg["vocab"]) for i in local_items}
    t0 = time.perf_counter()
    for s in range(0, len(local_items), 1024):
        ids = local_items[s:s + 1024]
        bat.bat_kv_prefill_entities(pool.handle, model.handle, bat.BAT_ENT_ITEM, ids, [item_toks[i] for i in ids],
                                    0, stream=stream)
    torch.cuda.synchronize()
    t_corpus = time.perf_counter() - t0
    if world > 1:
        bdist.exchange_remote(pool.handle, owner, rank, world)
        dist.barrier()

    # ---- batches
    rng = np.random.default_rng([args.seed, rank])
    n_batches = max(1, args.plans)
    batches = [make_queries(args, cfg, rng, 10_000_000 * (rank + 1) + 100_000 * k, args.batch, zipf_p)
               for k in range(n_batches)]
    qarrays = [bat.QueryArray(b) for b in batches]
    cold_ids = [bdist.cold_items(b, owner, rank) for b in batches]

    def fetch(k):
        return bdist.fetch_cold(pool.handle, cold_ids[k], stream) if world > 1 else 0

    def drop(k):
        if world > 1:
            bdist.drop_fetched(pool.handle, cold_ids[k])

    B = args.batch
    n_max = args.n_items
    hidden = torch.empty(B, cfg["hidden"], device=dev)
    labels_h = [torch.tensor(np.stack([q.labels for q in b]), dtype=torch.int32).pin_memory() for b in batches]
    labels_d = [l.to(dev) for l in labels_h]
    n_items_d = torch.full((B,), args.n_items, dtype=torch.int32, device=dev)
    scores = torch.empty(B, n_max, device=dev)
    topk = torch.empty(B, 10, dtype=torch.int32, device=dev)
    scores_h = torch.empty(B, n_max).pin_memory()
    topk_h = torch.empty(B, 10, dtype=torch.int32).pin_memory()

    # plan info (suffix tokens, visible pairs) for the FLOP count
    plans = []
    info = []
    for k in range(n_batches):
        fetch(k)
        plans.append(bat.bat_plan_build(pool.handle, model.handle, qarrays[k], stream))
        pi = bat.bat_plan_create(pool.handle, cfg["q_heads"] // cfg["kv_heads"], qarrays[k])
        info.append([bat.bat_plan_query_info(pi, b) for b in range(B)])
        bat.bat_plan_destroy(pi)
    # NOTE: for N > 1 the device plans reference fetched pages; they stay resident (no drop)
    flops_step = []
    toks_step = []
    for inf in info:
        f = 0.0
        for r in inf:
            # the last layer's attention covers only the last q-tile's rows (a8)
            f += algorithmic_flops_per_request(cfg, r["S"], r["n_live_pairs"], r["n_live_pairs_last"])[0]
        flops_step.append(f)
        toks_step.append(sum(r["S"] for r in inf))

    def step_device(k):
        bat.bat_prefill_plan(pool.handle, model.handle, plans[k % n_batches], hidden, stream)
        bat.bat_score(model.handle, hidden, labels_d[k % n_batches], n_items_d, B, n_max, scores, 10, topk, stream)

    # ---- device-resident timing
    for i in range(args.warmup):
        step_device(i)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    bat.bat_profile_reset(model.handle)
    bat.bat_profile_enable(model.handle, True)
    clk = ClockSampler(local)
    clk.start()
    n_launch0 = bat.bat_kernel_launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    prof_range = os.environ.get("BAT_PROFILE_RANGE") == "1"  # ncu --profile-from-start off
    torch.cuda.synchronize()
    if prof_range:
        torch.cuda.cudart().cudaProfilerStart()
    ev0.record(stream)
    for i in range(args.steps):
        step_device(i)
    ev1.record(stream)
    torch.cuda.synchronize()
    if prof_range:
        torch.cuda.cudart().cudaProfilerStop()
    launches = bat.bat_kernel_launch_count() - n_launch0
    clocks = clk.stop()
    bat.bat_profile_enable(model.handle, False)
    prof = bat.bat_profile_read(model.handle)
    ms = ev0.elapsed_time(ev1)
    if world > 1:
        t = torch.tensor([ms], device=red_dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    ms_step = ms / args.steps
    total_req = args.steps * B * world
    value = total_req / (ms / 1e3)
    alg_flops = sum(flops_step[i % n_batches] for i in range(args.steps))
    sfx_tokens = sum(toks_step[i % n_batches] for i in range(args.steps))

    # ---- end-to-end through the public call with host inputs
    for k in range(n_batches):
        bat.bat_plan_destroy(plans[k])
    h2d = d2h = 0
    for i in range(args.warmup):
        k = i % n_batches
        bat.bat_bipartite_prefill(pool.handle, model.handle, qarrays[k], hidden, stream)
    torch.cuda.synchronize()
    if world > 1:  # release every pulled copy once (batches share cold items)
        all_cold = np.unique(np.concatenate([c for c in cold_ids] + [np.zeros(0, np.int64)]))
        bdist.drop_fetched(pool.handle, all_cold)
        dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for i in range(args.steps):
        k = i % n_batches
        nf = fetch(k)
        bat.bat_bipartite_prefill(pool.handle, model.handle, qarrays[k], hidden, stream)
        lab = labels_h[k].to(dev, non_blocking=True)
        bat.bat_score(model.handle, hidden, lab, n_items_d, B, n_max, scores, 10, topk, stream)
        scores_h.copy_(scores, non_blocking=True)
        topk_h.copy_(topk, non_blocking=True)
        if i == 0:
            # plan image uploaded by the call + labels; results read back
            h2d = sum(4 * (2 * r["S"] + 8) for r in info[k]) + lab.numel() * 4
            d2h = scores_h.numel() * 4 + topk_h.numel() * 4
        if world > 1:
            torch.cuda.current_stream(dev).synchronize()
            drop(k)
    e1.record(stream)
    torch.cuda.synchronize()
    ems = e0.elapsed_time(e1)
    if world > 1:
        t = torch.tensor([ems], device=red_dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ems = float(t.item())
    e2e = total_req / (ems / 1e3)

    # ---- roofline of the dominant kernel (largest share of the step)
    dom = max(prof, key=lambda k: prof[k]["ms"])
    dp = prof[dom]
    achieved = dp["flops"] / (dp["ms"] / 1e3) / 1e12 if dp["ms"] > 0 else 0.0
    traffic = None
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp) and B == 64:  # captured at this batch (layer-0 launch, one ncu --set full)
        traffic = json.load(open(tp))["dram_bytes_per_launch"].get(dom)
    roof = dict(kernel=dom, bound="tensor", achieved=achieved, peak=pk["bf16_sus"], unit="TFLOP/s",
                frac=achieved / pk["bf16_sus"], traffic=traffic,
                traffic_unit="DRAM bytes per launch (ncu dram__bytes_read.sum + dram__bytes_write.sum)",
                algorithmic_bytes_per_launch=dp["bytes"] / max(1, dp["launches"]),
                peak_note=f"bf16 sustained, {pk['src']} (kernel timed inside the step)",
                share_of_step=dp["ms"] / max(1e-9, sum(v["ms"] for v in prof.values())))
    at = prof["attention"]
    attn_ach = at["flops"] / (at["ms"] / 1e3) / 1e12 if at["ms"] > 0 else 0.0
    kernels = {k: dict(ms_per_step=v["ms"] / args.steps, launches_per_step=v["launches"] / args.steps,
                       tflops=(v["flops"] / (v["ms"] / 1e3) / 1e12) if v["ms"] > 0 and v["flops"] > 0 else None,
                       gbs=(v["bytes"] / (v["ms"] / 1e3) / 1e9) if v["ms"] > 0 else None)
               for k, v in prof.items() if v["launches"]}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        t_req, sample, threads, _ = oracle_time_per_request(args, args.cpu_budget)
        cpu = dict(value=1.0 / t_req, unit="requests/s", cores=threads, kind="oracle", sample=sample)

    if rank == 0:
        line = dict(
            metric=METRIC, value=value, unit="requests/s", n_gpus=world, steps=args.steps, warmup=args.warmup,
            ms_per_step=ms_step, higher_is_better=True, scaling="weak", vs_baseline=None, dtype="bf16",
            data="synthetic (random-init weights, seeded synthetic requests; item KV computed by the model)",
            config=dict(workload=WORKLOAD if args.model == "qwen2-1.5b" else
                        f"{args.model}-shaped, 1 user of {args.n_user} tokens + {args.n_items} items of "
                        f"{args.item_len} tokens, bf16, item-as-prefix", batch_per_gpu=B, global_batch=B * world, seq_len=args.n_user + args.n_items * args.item_len + args.n_instr,
                        suffix_tokens_per_request=args.n_user + args.n_instr, prefix_tokens_per_request=args.n_items * args.item_len,
                        corpus_items=args.corpus, item_hotness="Zipf s=1.093", parallelism=f"dp{world}",
                        hrcs=dict(replication_ratio=r_rep, r_max=r_max, alpha=args.alpha, t_request_s=0.0015,
                                  link_gbs=770.0, cold_items_per_step=float(np.mean([len(c) for c in cold_ids])))
                        if world > 1 else None,
                        l2="inputs larger than L2 (2.6 GB of weights streamed every step)"),
            prefill_tokens_per_s=sfx_tokens * world / (ms / 1e3),
            served_tokens_per_s=total_req * (args.n_user + args.n_instr + args.n_items * args.item_len) / (ms / 1e3),
            algorithmic_tflops=alg_flops * world / (ms / 1e3) / 1e12,
            mfu=dict(of_measured_burst=alg_flops / (ms / 1e3) / 1e12 / pk["bf16"],
                     of_measured_sustained=alg_flops / (ms / 1e3) / 1e12 / pk["bf16_sus"],
                     of_spec_2250=alg_flops / (ms / 1e3) / 1e12 / 2250.0),
            roofline=roof,
            attention=dict(tflops=attn_ach, frac_of_sustained=attn_ach / pk["bf16_sus"],
                           frac_of_burst=attn_ach / pk["bf16"], ms_per_step=at["ms"] / args.steps),
            kernels=kernels,
            e2e=dict(value=e2e, unit="requests/s", h2d_bytes_per_step=h2d, d2h_bytes_per_step=d2h),
            gpu_launches=launches,
            clocks=clocks,
            cpu_baseline=cpu,
            corpus_prefill_s=t_corpus,
        )
        print(json.dumps(line))
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()

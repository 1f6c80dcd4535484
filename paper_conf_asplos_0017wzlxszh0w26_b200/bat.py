"""ctypes binding of libbat.so (include/bat.h) — argument marshalling only.

Every function here has the name of the C entry point it calls and does no arithmetic of
the method: it packs Python/numpy arguments into the C structs, calls the library, checks
the status and raises ``BatError`` with ``bat_last_error()``.  All computation of the
bipartite prefill runs in the library's sm_100a kernels; there is no CPU fallback — if the
shared library is missing this module raises on first use.

PyTorch is used by callers only for device memory and streams: device pointers are passed
as integers (``tensor.data_ptr()``) and streams as ``torch.cuda.Stream.cuda_stream``.
"""
from __future__ import annotations

import ctypes
import os
from ctypes import (POINTER, Structure, byref, c_char_p, c_double, c_float, c_int32, c_int64,
                    c_size_t, c_uint8, c_void_p)
from typing import List, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("BAT_LIB") or os.path.join(_HERE, "libbat.so")  # BAT_LIB: experiment builds

BAT_OK = 0
BAT_BF16, BAT_FP32 = 0, 1
BAT_ENT_USER, BAT_ENT_ITEM, BAT_ENT_HEADER = 0, 1, 2
BAT_ORDER_UP, BAT_ORDER_IP = 0, 1
BAT_PF_TOKENS, BAT_PF_POS, BAT_PF_SEG, BAT_PF_PAGES, BAT_PF_VALID, BAT_PF_KSEG, BAT_PF_KORD, BAT_PF_TILES, BAT_PF_DISC = range(9)
STATUS_NAMES = {0: "BAT_OK", -1: "BAT_E_INVAL", -2: "BAT_E_OOM", -3: "BAT_E_CUDA",
                -4: "BAT_E_NOTFOUND", -5: "BAT_E_POOLFULL", -6: "BAT_E_UNSUPPORTED",
                -7: "BAT_E_STATE"}


class BatError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


class bat_model_cfg(Structure):
    _fields_ = [("layers", c_int32), ("hidden", c_int32), ("q_heads", c_int32),
                ("kv_heads", c_int32), ("head_dim", c_int32), ("ffn", c_int32),
                ("vocab", c_int32), ("rope_theta", c_float), ("rms_eps", c_float),
                ("dtype", c_int32)]


class bat_pool_cfg(Structure):
    _fields_ = [("device", c_int32), ("page_tokens", c_int32), ("num_pages", c_int64),
                ("dtype", c_int32), ("layers", c_int32), ("kv_heads", c_int32),
                ("head_dim", c_int32), ("rank", c_int32), ("world", c_int32)]


class bat_query(Structure):
    _fields_ = [("order", c_int32), ("use_cache", c_int32), ("user_id", c_int64),
                ("user_tok", POINTER(c_int32)), ("n_user", c_int32), ("n_items", c_int32),
                ("item_id", POINTER(c_int64)), ("item_off", POINTER(c_int32)),
                ("item_tok", POINTER(c_int32)), ("instr_tok", POINTER(c_int32)),
                ("n_instr", c_int32), ("header_id", c_int64), ("header_tok", POINTER(c_int32)),
                ("n_header", c_int32), ("multi_disc", c_int32), ("pic_tail", c_int32)]


_lib = None


class bat_sched_cfg(Structure):
    _fields_ = [("policy", c_int32), ("capacity_pages", c_int64), ("window", c_double)]


class bat_sched_decision(Structure):
    _fields_ = [("order", c_int32), ("user_hit", c_int32), ("admit", c_int32), ("n_evict", c_int32),
                ("freq", c_int32)]


BAT_SCHED_HOTNESS, BAT_SCHED_GREEDY, BAT_SCHED_UP, BAT_SCHED_IP, BAT_SCHED_RE = range(5)
SCHED_POLICY = {"hotness": BAT_SCHED_HOTNESS, "greedy": BAT_SCHED_GREEDY, "up": BAT_SCHED_UP,
                "ip": BAT_SCHED_IP, "re": BAT_SCHED_RE}


def lib() -> ctypes.CDLL:
    """Load libbat.so (fails loudly when the extension has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"libbat.so not built ({LIB_PATH}); run __graft_entry__.build()")
    L = ctypes.CDLL(LIB_PATH)
    S = c_int32  # bat_status
    sig = {
        "bat_last_error": (c_char_p, []),
        "bat_version": (c_char_p, []),
        "bat_kernel_launch_count": (c_int64, []),
        "bat_model_create": (S, [POINTER(bat_model_cfg), POINTER(c_void_p), c_int32, c_int32, POINTER(c_void_p)]),
        "bat_model_destroy": (S, [c_void_p]),
        "bat_kv_pool_create": (S, [POINTER(bat_pool_cfg), POINTER(c_void_p)]),
        "bat_kv_pool_destroy": (S, [c_void_p]),
        "bat_kv_page_bytes": (c_int64, [c_void_p]),
        "bat_kv_pool_stats": (S, [c_void_p, POINTER(c_int64), POINTER(c_int64), POINTER(c_int64)]),
        "bat_kv_append": (S, [c_void_p, c_int32, c_int64, c_void_p, c_void_p, c_int32, c_void_p]),
        "bat_kv_reserve": (S, [c_void_p, c_int32, c_int64, c_int32]),
        "bat_kv_evict": (S, [c_void_p, c_int32, c_int64]),
        "bat_kv_lookup": (S, [c_void_p, c_int32, c_int64, POINTER(c_int32), POINTER(c_int32), c_int32, POINTER(c_int32)]),
        "bat_kv_read": (S, [c_void_p, c_int32, c_int64, c_void_p, c_void_p, c_void_p]),
        "bat_kv_prefill_entities": (S, [c_void_p, c_void_p, c_int32, c_int32, POINTER(c_int64), POINTER(c_int32),
                                        POINTER(c_int32), c_int32, c_int32, c_int64, c_void_p]),
        "bat_bipartite_prefill": (S, [c_void_p, c_void_p, POINTER(bat_query), c_int32, c_void_p, c_void_p]),
        "bat_score": (S, [c_void_p, c_void_p, c_void_p, c_void_p, c_int32, c_int32, c_void_p, c_int32, c_void_p,
                          c_void_p, c_void_p]),
        "bat_plan_create": (S, [c_void_p, c_int32, POINTER(bat_query), c_int32, POINTER(c_void_p)]),
        "bat_plan_destroy": (S, [c_void_p]),
        "bat_plan_query_info": (S, [c_void_p, c_int32, POINTER(c_int64)]),
        "bat_plan_export": (S, [c_void_p, c_int32, c_int32, POINTER(c_int32), c_int64, POINTER(c_int64)]),
        "bat_hrcs_rmax": (S, [c_double, c_double, c_double, c_int32, c_double, c_int32, POINTER(c_double)]),
        "bat_hrcs_place": (S, [POINTER(c_double), c_int64, c_double, c_int32, POINTER(c_int32), POINTER(c_double)]),
        "bat_pool_ipc_handle": (S, [c_void_p, c_void_p]),
        "bat_pool_attach_peer": (S, [c_void_p, c_int32, c_void_p]),
        "bat_kv_register_remote": (S, [c_void_p, c_int32, c_int64, c_int32, POINTER(c_int32), c_int32, c_int32]),
        "bat_kv_lookup_remote": (S, [c_void_p, c_int32, c_int64, POINTER(c_int32), POINTER(c_int32),
                                     POINTER(c_int32), c_int32, POINTER(c_int32)]),
        "bat_kv_fetch": (S, [c_void_p, c_int32, POINTER(c_int64), c_int32, POINTER(c_int32), c_void_p]),
        "bat_plan_build": (S, [c_void_p, c_void_p, POINTER(bat_query), c_int32, c_void_p, POINTER(c_void_p)]),
        "bat_prefill_plan": (S, [c_void_p, c_void_p, c_void_p, c_void_p, c_void_p]),
        "bat_profile_enable": (S, [c_void_p, c_int32]),
        "bat_profile_read": (S, [c_void_p, c_int32, POINTER(c_double), POINTER(c_int64), POINTER(c_double),
                                 POINTER(c_double)]),
        "bat_profile_reset": (S, [c_void_p]),
        "bat_debug_attach_peer_pool": (S, [c_void_p, c_int32, c_void_p]),
        "bat_debug_gemm": (S, [c_int32, c_int32, c_int32, c_int32, c_void_p, c_void_p, c_int64, c_void_p,
                               c_int32, c_void_p, c_int32, c_int32, c_void_p]),
        "bat_debug_attention_layer": (S, [c_void_p, c_void_p, POINTER(bat_query), c_int32, c_int32, c_void_p,
                                          c_void_p, c_int32, c_void_p]),
        "bat_score_multi": (S, [c_void_p, c_void_p, c_void_p, c_void_p, c_int32, c_int32, c_void_p, c_int32, c_void_p,
                                c_void_p, c_void_p]),
        "bat_plan_export_device": (S, [c_void_p, c_int32, c_int32, c_void_p, c_int64, POINTER(c_int64)]),
        "bat_kv_release": (S, [c_void_p, c_int32, POINTER(c_int64), c_int32, c_void_p]),
        "bat_kv_staging_reserve": (S, [c_void_p, c_int32, c_int64]),
        "bat_plan_build_staged": (S, [c_void_p, c_void_p, POINTER(bat_query), c_int32, c_int32, c_void_p,
                                      POINTER(c_void_p)]),
        "bat_plan_fetch": (S, [c_void_p, c_void_p, POINTER(c_int64), c_void_p]),
        "bat_plan_bytes": (S, [c_void_p, POINTER(c_int64), POINTER(c_int64)]),
        "bat_plan_work_info": (S, [c_void_p, POINTER(c_int64)]),
        "bat_hrcs_refresh": (S, [POINTER(c_int32), c_int64, POINTER(c_double), c_int64, c_double, c_int32,
                                 POINTER(c_int32)]),
        "bat_kv_replicate": (S, [c_void_p, c_int32, POINTER(c_int64), c_int32, c_void_p]),
        "bat_sched_create": (S, [POINTER(bat_sched_cfg), POINTER(c_void_p)]),
        "bat_sched_destroy": (S, [c_void_p]),
        "bat_sched_decide": (S, [c_void_p, c_double, c_int64, c_int32, c_int32, POINTER(bat_sched_decision),
                                 POINTER(c_int64), c_int32]),
        "bat_sched_stats": (S, [c_void_p, POINTER(c_int64)]),
        "bat_sched_is_cached": (c_int32, [c_void_p, c_int64]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


EXPORTED = ("bat_last_error", "bat_version", "bat_kernel_launch_count", "bat_model_create",
            "bat_model_destroy", "bat_kv_pool_create", "bat_kv_pool_destroy", "bat_kv_page_bytes",
            "bat_kv_pool_stats", "bat_kv_append", "bat_kv_reserve", "bat_kv_evict", "bat_kv_lookup",
            "bat_kv_read", "bat_kv_prefill_entities", "bat_bipartite_prefill", "bat_score",
            "bat_plan_create", "bat_plan_destroy", "bat_plan_query_info", "bat_plan_export",
            "bat_hrcs_rmax", "bat_hrcs_place", "bat_pool_ipc_handle", "bat_pool_attach_peer",
            "bat_kv_register_remote", "bat_kv_lookup_remote", "bat_kv_fetch", "bat_debug_gemm", "bat_debug_attention_layer",
            "bat_plan_build", "bat_prefill_plan", "bat_profile_enable", "bat_profile_read",
            "bat_profile_reset", "bat_debug_attach_peer_pool", "bat_sched_create", "bat_sched_destroy",
            "bat_sched_decide", "bat_sched_stats", "bat_sched_is_cached", "bat_score_multi",
            "bat_plan_export_device", "bat_kv_release", "bat_kv_staging_reserve", "bat_plan_build_staged",
            "bat_plan_fetch", "bat_plan_bytes", "bat_hrcs_refresh", "bat_kv_replicate",
            "bat_plan_work_info")


def _check(status: int) -> None:
    if status != BAT_OK:
        raise BatError(status, lib().bat_last_error().decode())


def _i32p(a: np.ndarray):
    return a.ctypes.data_as(POINTER(c_int32))


def _i64p(a: np.ndarray):
    return a.ctypes.data_as(POINTER(c_int64))


def _vp(x) -> Optional[int]:
    """device pointer / stream handle as int (accepts torch tensors / streams, ints, None)."""
    if x is None:
        return None
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if hasattr(x, "cuda_stream"):
        return x.cuda_stream
    return int(x)


# ----------------------------------------------------------------------------- misc
def bat_last_error() -> str:
    return lib().bat_last_error().decode()


def bat_version() -> str:
    return lib().bat_version().decode()


def bat_kernel_launch_count() -> int:
    return int(lib().bat_kernel_launch_count())


# ---------------------------------------------------------------------------- model
def model_cfg(cfg: dict, dtype: int = BAT_BF16) -> bat_model_cfg:
    return bat_model_cfg(cfg["layers"], cfg["hidden"], cfg["q_heads"], cfg["kv_heads"],
                         cfg["head_dim"], cfg["ffn"], cfg["vocab"], float(cfg["rope_theta"]),
                         float(cfg["rms_eps"]), dtype)


def bat_model_create(cfg: dict, weight_ptrs: Sequence[int], device: int = 0,
                     dtype: int = BAT_BF16) -> int:
    c = model_cfg(cfg, dtype)
    arr = (c_void_p * len(weight_ptrs))(*[int(p) for p in weight_ptrs])
    out = c_void_p()
    _check(lib().bat_model_create(byref(c), arr, len(weight_ptrs), device, byref(out)))
    return out.value


def bat_model_destroy(model: int) -> None:
    _check(lib().bat_model_destroy(model))


# ----------------------------------------------------------------------------- pool
def bat_kv_pool_create(device: int, num_pages: int, layers: int, kv_heads: int, head_dim: int,
                       dtype: int = BAT_BF16, rank: int = 0, world: int = 1,
                       page_tokens: int = 16) -> int:
    c = bat_pool_cfg(device, page_tokens, num_pages, dtype, layers, kv_heads, head_dim, rank, world)
    out = c_void_p()
    _check(lib().bat_kv_pool_create(byref(c), byref(out)))
    return out.value


def bat_kv_pool_destroy(pool: int) -> None:
    _check(lib().bat_kv_pool_destroy(pool))


def bat_kv_page_bytes(pool: int) -> int:
    return int(lib().bat_kv_page_bytes(pool))


def bat_kv_pool_stats(pool: int):
    f, u, n = c_int64(), c_int64(), c_int64()
    _check(lib().bat_kv_pool_stats(pool, byref(f), byref(u), byref(n)))
    return f.value, u.value, n.value


def bat_kv_append(pool: int, kind: int, id_: int, k, v, n_tokens: int, stream=None) -> None:
    _check(lib().bat_kv_append(pool, kind, id_, _vp(k), _vp(v), n_tokens, _vp(stream)))


def bat_kv_reserve(pool: int, kind: int, id_: int, n_tokens: int) -> None:
    _check(lib().bat_kv_reserve(pool, kind, id_, n_tokens))


def bat_kv_evict(pool: int, kind: int, id_: int) -> None:
    _check(lib().bat_kv_evict(pool, kind, id_))


def bat_kv_lookup(pool: int, kind: int, id_: int):
    n_tok, n_pg = c_int32(), c_int32()
    _check(lib().bat_kv_lookup(pool, kind, id_, byref(n_tok), None, 0, byref(n_pg)))
    pages = np.zeros(max(n_pg.value, 1), dtype=np.int32)
    _check(lib().bat_kv_lookup(pool, kind, id_, byref(n_tok), _i32p(pages), len(pages), byref(n_pg)))
    return n_tok.value, pages[: n_pg.value]


def bat_kv_read(pool: int, kind: int, id_: int, k_out, v_out, stream=None) -> None:
    _check(lib().bat_kv_read(pool, kind, id_, _vp(k_out), _vp(v_out), _vp(stream)))


def bat_kv_prefill_entities(pool: int, model: int, kind: int, ids: Sequence[int],
                            token_lists: Sequence[np.ndarray], pos0: int = 0,
                            ctx_kind: int = -1, ctx_id: int = 0, stream=None) -> None:
    ids_a = np.ascontiguousarray(ids, dtype=np.int64)
    off = np.zeros(len(token_lists) + 1, dtype=np.int32)
    off[1:] = np.cumsum([len(t) for t in token_lists])
    toks = np.ascontiguousarray(np.concatenate([np.asarray(t, np.int32) for t in token_lists]), dtype=np.int32)
    _check(lib().bat_kv_prefill_entities(pool, model, kind, len(ids_a), _i64p(ids_a), _i32p(off),
                                         _i32p(toks), pos0, ctx_kind, ctx_id, _vp(stream)))


# -------------------------------------------------------------------------- queries
class QueryArray:
    """A bat_query[B] built from request descriptions (objects with user_id, user_tok,
    item_ids, item_toks, instr_tok, order "UP"/"IP", use_cache, header_id, header_tok);
    owns the host arrays the structs point to."""

    def __init__(self, queries):
        self._keep: List[np.ndarray] = []
        self.arr = (bat_query * len(queries))()
        for b, q in enumerate(queries):
            keep = lambda a, dt: self._keep.append(np.ascontiguousarray(a, dtype=dt)) or self._keep[-1]
            ut = keep(q.user_tok, np.int32)
            iid = keep(q.item_ids, np.int64)
            off = np.zeros(len(q.item_toks) + 1, dtype=np.int32)
            off[1:] = np.cumsum([len(t) for t in q.item_toks])
            off = keep(off, np.int32)
            it = keep(np.concatenate([np.asarray(t, np.int32) for t in q.item_toks]), np.int32)
            xt = keep(q.instr_tok, np.int32)
            ht = keep(q.header_tok if len(q.header_tok) else np.zeros(1, np.int32), np.int32)
            s = self.arr[b]
            s.order = BAT_ORDER_UP if q.order == "UP" else BAT_ORDER_IP
            s.use_cache = 1 if q.use_cache else 0
            s.user_id = int(q.user_id)
            s.user_tok = _i32p(ut)
            s.n_user = len(q.user_tok)
            s.n_items = len(q.item_ids)
            s.item_id = _i64p(iid)
            s.item_off = _i32p(off)
            s.item_tok = _i32p(it)
            s.instr_tok = _i32p(xt)
            s.n_instr = len(q.instr_tok)
            s.header_id = int(getattr(q, "header_id", 0))
            s.header_tok = _i32p(ht)
            s.n_header = len(q.header_tok)
            s.multi_disc = 1 if getattr(q, "multi_disc", False) else 0
            s.pic_tail = int(getattr(q, "pic_tail", 0) or 0)

    def __len__(self):
        return len(self.arr)


def bat_bipartite_prefill(pool: int, model: int, queries: QueryArray, out_hidden, stream=None) -> None:
    _check(lib().bat_bipartite_prefill(pool, model, queries.arr, len(queries), _vp(out_hidden), _vp(stream)))


def bat_score(model: int, hidden, labels, n_items, B: int, n_max: int, scores, k: int = 0,
              topk=None, stream=None, logits=None) -> None:
    _check(lib().bat_score(model, _vp(hidden), _vp(labels), _vp(n_items), B, n_max, _vp(scores),
                           k, _vp(topk), _vp(logits), _vp(stream)))


def bat_score_multi(model: int, hidden, labels, n_items, B: int, n_max: int, scores, k: int = 0,
                    topk=None, stream=None, logits=None) -> None:
    _check(lib().bat_score_multi(model, _vp(hidden), _vp(labels), _vp(n_items), B, n_max, _vp(scores),
                                 k, _vp(topk), _vp(logits), _vp(stream)))


# ----------------------------------------------------------------------------- plan
def bat_plan_create(pool: int, group: int, queries: QueryArray) -> int:
    out = c_void_p()
    _check(lib().bat_plan_create(pool, group, queries.arr, len(queries), byref(out)))
    return out.value


def bat_plan_destroy(plan: int) -> None:
    _check(lib().bat_plan_destroy(plan))


PLAN_INFO_KEYS = ("S", "P", "n_pages", "n_prefix_pages", "n_qtiles", "n_ktiles", "token_off",
                  "scratch0", "n_live_pairs", "qtile_tokens", "qtile0", "page_off", "n_live_pairs_last")


def bat_plan_query_info(plan: int, b: int) -> dict:
    info = (c_int64 * 13)()
    _check(lib().bat_plan_query_info(plan, b, info))
    return dict(zip(PLAN_INFO_KEYS, [int(x) for x in info]))


def bat_plan_export(plan: int, b: int, field: int) -> np.ndarray:
    n = c_int64()
    _check(lib().bat_plan_export(plan, b, field, None, 0, byref(n)))
    out = np.zeros(max(n.value, 1), dtype=np.int32)
    _check(lib().bat_plan_export(plan, b, field, _i32p(out), len(out), byref(n)))
    return out[: n.value]


BAT_PFD_VIS, BAT_PFD_VIS_LAST, BAT_PFD_KPAGES, BAT_PFD_STAGE = range(4)
BAT_PFD_NOT_LOADED = -2147483647


def bat_plan_export_device(plan: int, b: int, field: int) -> np.ndarray:
    """The device image of a bat_plan_build plan decoded as the attention kernel reads it:
    VIS / VIS_LAST uint8 [S][n_ktiles*128]; KPAGES int32 [n_ktiles*8]; STAGE int32 [S][3]."""
    n = c_int64()
    _check(lib().bat_plan_export_device(plan, b, field, None, 0, byref(n)))
    out = np.zeros(max(n.value, 1), dtype=np.int32 if field in (BAT_PFD_KPAGES, BAT_PFD_STAGE) else np.uint8)
    _check(lib().bat_plan_export_device(plan, b, field, out.ctypes.data_as(c_void_p), len(out), byref(n)))
    return out[: n.value]


# ---------------------------------------------------------------- planned execution
def bat_plan_build(pool: int, model: int, queries: QueryArray, stream=None) -> int:
    out = c_void_p()
    _check(lib().bat_plan_build(pool, model, queries.arr, len(queries), _vp(stream), byref(out)))
    return out.value


def bat_prefill_plan(pool: int, model: int, plan: int, out_hidden, stream=None) -> None:
    _check(lib().bat_prefill_plan(pool, model, plan, _vp(out_hidden), _vp(stream)))


# ------------------------------------------------------------------------ profiling
K_CLASSES = ("embed", "rmsnorm", "gemm_qkv", "stage", "attention", "gemm_o", "gemm_gate_up",
             "gemm_down", "other")


def bat_profile_enable(model: int, on: bool = True) -> None:
    _check(lib().bat_profile_enable(model, 1 if on else 0))


def bat_profile_read(model: int) -> dict:
    out = {}
    for i, name in enumerate(K_CLASSES):
        ms, n, fl, by = c_double(), c_int64(), c_double(), c_double()
        _check(lib().bat_profile_read(model, i, byref(ms), byref(n), byref(fl), byref(by)))
        out[name] = dict(ms=ms.value, launches=n.value, flops=fl.value, bytes=by.value)
    return out


def bat_profile_reset(model: int) -> None:
    _check(lib().bat_profile_reset(model))


# ------------------------------------------------------------------- HRCS / multi-GPU
def bat_hrcs_rmax(B: float, t: float, alpha: float, c: int, tau_i: float, N: int) -> float:
    out = c_double()
    _check(lib().bat_hrcs_rmax(B, t, alpha, c, tau_i, N, byref(out)))
    return out.value


def bat_hrcs_place(freq: Sequence[float], r_max: float, world: int):
    f = np.ascontiguousarray(freq, dtype=np.float64)
    owner = np.zeros(len(f), dtype=np.int32)
    r = c_double()
    _check(lib().bat_hrcs_place(f.ctypes.data_as(POINTER(c_double)), len(f), r_max, world,
                                _i32p(owner), byref(r)))
    return r.value, owner


def bat_hrcs_refresh(owner_old: Sequence[int], freq_new: Sequence[float], r: float, world: int) -> np.ndarray:
    o = np.ascontiguousarray(owner_old, dtype=np.int32)
    f = np.ascontiguousarray(freq_new, dtype=np.float64)
    out = np.zeros(len(f), dtype=np.int32)
    _check(lib().bat_hrcs_refresh(_i32p(o) if len(o) else None, len(o), f.ctypes.data_as(POINTER(c_double)), len(f),
                                  r, world, _i32p(out)))
    return out


def bat_kv_replicate(pool: int, kind: int, ids: Sequence[int], stream=None) -> None:
    a = np.ascontiguousarray(ids, dtype=np.int64)
    _check(lib().bat_kv_replicate(pool, kind, _i64p(a), len(a), _vp(stream)))


def bat_pool_ipc_handle(pool: int) -> bytes:
    buf = (c_uint8 * 64)()
    _check(lib().bat_pool_ipc_handle(pool, buf))
    return bytes(buf)


def bat_pool_attach_peer(pool: int, peer: int, handle: bytes) -> None:
    buf = (c_uint8 * 64).from_buffer_copy(handle)
    _check(lib().bat_pool_attach_peer(pool, peer, buf))


def bat_kv_register_remote(pool: int, kind: int, id_: int, owner: int, pages: Sequence[int],
                           n_tokens: int) -> None:
    pg = np.ascontiguousarray(pages, dtype=np.int32)
    _check(lib().bat_kv_register_remote(pool, kind, id_, owner, _i32p(pg), len(pg), n_tokens))


def bat_kv_lookup_remote(pool: int, kind: int, id_: int):
    owner, n_tok, n_pg = c_int32(), c_int32(), c_int32()
    _check(lib().bat_kv_lookup_remote(pool, kind, id_, byref(owner), byref(n_tok), None, 0, byref(n_pg)))
    pages = np.zeros(max(n_pg.value, 1), dtype=np.int32)
    _check(lib().bat_kv_lookup_remote(pool, kind, id_, byref(owner), byref(n_tok), _i32p(pages), len(pages),
                                      byref(n_pg)))
    return owner.value, n_tok.value, pages[: n_pg.value]


def bat_kv_fetch(pool: int, kind: int, ids: Sequence[int], stream=None) -> int:
    a = np.ascontiguousarray(ids, dtype=np.int64)
    n = c_int32()
    _check(lib().bat_kv_fetch(pool, kind, _i64p(a), len(a), byref(n), _vp(stream)))
    return n.value


def bat_kv_release(pool: int, kind: int, ids: Sequence[int], stream=None) -> None:
    a = np.ascontiguousarray(ids, dtype=np.int64)
    _check(lib().bat_kv_release(pool, kind, _i64p(a), len(a), _vp(stream)))


def bat_kv_staging_reserve(pool: int, n_slots: int, pages_per_slot: int) -> None:
    _check(lib().bat_kv_staging_reserve(pool, n_slots, pages_per_slot))


def bat_plan_build_staged(pool: int, model: int, queries: QueryArray, slot: int, stream=None) -> int:
    out = c_void_p()
    _check(lib().bat_plan_build_staged(pool, model, queries.arr, len(queries), slot, _vp(stream), byref(out)))
    return out.value


def bat_plan_bytes(plan: int):
    """(host image bytes uploaded per call, device image bytes)"""
    h, d = c_int64(), c_int64()
    _check(lib().bat_plan_bytes(plan, byref(h), byref(d)))
    return h.value, d.value


def bat_plan_work_info(plan: int) -> dict:
    out = (c_int64 * 6)()
    _check(lib().bat_plan_work_info(plan, out))
    return dict(zip(("n_work", "n_work_last", "split_groups", "split_slots", "split_groups_last",
                     "split_slots_last"), [int(x) for x in out]))


def bat_plan_fetch(pool: int, plan: int, stream=None) -> int:
    n = c_int64()
    _check(lib().bat_plan_fetch(pool, plan, byref(n), _vp(stream)))
    return n.value


# ------------------------------------------------------------------------ test-only
def bat_debug_gemm(epi: int, M: int, N: int, K: int, A, Bw, b_rows: int, out, ldo: int,
                   bias=None, up_row0: int = 0, device: int = 0, stream=None) -> None:
    _check(lib().bat_debug_gemm(epi, M, N, K, _vp(A), _vp(Bw), b_rows, _vp(out), ldo, _vp(bias),
                                up_row0, device, _vp(stream)))


def bat_debug_attention_layer(pool: int, model: int, queries: QueryArray, layer: int, qkv, out_o,
                              rope_enabled: bool = True, stream=None) -> None:
    _check(lib().bat_debug_attention_layer(pool, model, queries.arr, len(queries), layer, _vp(qkv),
                                           _vp(out_o), 1 if rope_enabled else 0, _vp(stream)))


def bat_debug_attach_peer_pool(pool: int, peer: int, other: int) -> None:
    _check(lib().bat_debug_attach_peer_pool(pool, peer, other))


# ------------------------------------------------------------------ prompt scheduler (NEXT-2)
def bat_sched_create(policy: str, capacity_pages: int, window: float) -> int:
    h = c_void_p()
    _check(lib().bat_sched_create(byref(bat_sched_cfg(SCHED_POLICY[policy], capacity_pages, window)), byref(h)))
    return h.value


def bat_sched_destroy(s: int) -> None:
    _check(lib().bat_sched_destroy(s))


def bat_sched_decide(s: int, t: float, user_id: int, tau_u: int, tau_i: int, evict_cap: int = 4096):
    """-> (order: "UP" | "IP" | "RE", user_hit, admit, evicted user ids, f_u)"""
    d = bat_sched_decision()
    ev = (c_int64 * max(1, evict_cap))()
    _check(lib().bat_sched_decide(s, t, user_id, tau_u, tau_i, byref(d), ev, evict_cap))
    order = {BAT_ORDER_UP: "UP", BAT_ORDER_IP: "IP"}.get(d.order, "RE")
    return order, bool(d.user_hit), bool(d.admit), [int(ev[i]) for i in range(d.n_evict)], d.freq


def bat_sched_stats(s: int) -> dict:
    out = (c_int64 * 7)()
    _check(lib().bat_sched_stats(s, out))
    return dict(tokens=out[0], reused=out[1], hits=out[2], up=out[3], ip=out[4], cached_users=out[5],
                used_pages=out[6])


def bat_sched_is_cached(s: int, user_id: int) -> bool:
    return bool(lib().bat_sched_is_cached(s, user_id))

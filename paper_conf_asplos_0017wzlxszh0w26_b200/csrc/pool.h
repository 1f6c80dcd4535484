// Disaggregated paged KV pool: one page arena per GPU, entries at
// user / item granularity, every entry a list of 16-token pages holding all layers.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <deque>
#include <string>
#include <unordered_map>
#include <vector>

#include "common.h"

namespace bat {

struct EntityKey {
  int32_t kind;
  int64_t id;
  bool operator==(const EntityKey& o) const { return kind == o.kind && id == o.id; }
};
struct EntityKeyHash {
  size_t operator()(const EntityKey& k) const {
    uint64_t x = static_cast<uint64_t>(k.id) * 0x9E3779B97F4A7C15ull ^ static_cast<uint64_t>(k.kind);
    x ^= x >> 29;
    return static_cast<size_t>(x * 0xBF58476D1CE4E5B9ull);
  }
};

struct Entity {
  int32_t n_tokens = 0;
  std::vector<int32_t> pages;
  bool fetched = false;  // a local copy of a remote (cold-sharded) entry
  int32_t pins = 0;      // live device plans referencing the pages (bat_plan_build)
  int32_t refs = 0;      // fetched copies: batches holding it (bat_kv_fetch / bat_kv_release)
};

struct RemoteEntity {
  int32_t owner = -1;
  int32_t n_tokens = 0;
  std::vector<int32_t> pages;  // page ids in the owner's arena
};

// Page layout (bf16): page = [layers][2 (K,V)][kv_heads][block], block = one head's 16 K (or
// V) rows of one layer = [2 slot groups][Dp/64 chunks][8 slots][64] with the 128-byte swizzle of
// the tensor-core operand layout inside each 1 KB atom: element (slot r, col c) sits at
// (r/8)*(Dp/64)*1024 + (c/64)*1024 + (r%8)*128 + ((((c%64)/8) ^ (r%8)) * 16) + (c%8)*2
// (ptx::page_blk_off).  A block is ONE contiguous bulk copy that lands in shared memory ready
// for tcgen05.mma (8-row-group stride (Dp/64) KB).
struct PageGeometry {
  int32_t layers = 0, kv_heads = 0, head_dim = 0, dpad = 0;
  int64_t block_bytes = 2048;  // [16][64] bf16
  int64_t head_bytes = 0;      // (dpad/64) blocks
  int64_t layer_bytes = 0;     // 2 * kv_heads * head_bytes
  int64_t page_bytes = 0;      // layers * layer_bytes
  bool f32 = false;            // BAT_FP32 pool: block = plain [16 slots][head_dim] fp32
  void init(int L, int hkv, int d, bool fp32 = false) {
    layers = L;
    kv_heads = hkv;
    head_dim = d;
    f32 = fp32;
    dpad = fp32 ? d : head_dim_pad(d);
    if (fp32) block_bytes = int64_t(16) * d * 4;
    head_bytes = fp32 ? block_bytes : (dpad / 64) * block_bytes;
    layer_bytes = 2 * kv_heads * head_bytes;
    page_bytes = layers * layer_bytes;
  }
};

struct Pool {
  bat_pool_cfg cfg{};
  bool index_only = false;
  int device = -1;
  PageGeometry geo;
  char* arena = nullptr;  // num_pages + 1 pages; page num_pages is the all-zero page
  int32_t zero_page = 0;
  std::vector<int32_t> free_pages;
  std::unordered_map<EntityKey, Entity, EntityKeyHash> index;
  std::unordered_map<EntityKey, RemoteEntity, EntityKeyHash> remote;
  std::vector<char*> peer_arena;  // by rank (IPC-mapped), nullptr for self / unattached
  std::vector<uint8_t> peer_ipc;  // 1 if peer_arena[r] came from cudaIpcOpenMemHandle
  uint64_t ipc_handle[8] = {0};
  // pinned staging of the fetch descriptors (bat_kv_fetch stays asynchronous on its stream)
  void* fetch_host = nullptr;
  size_t fetch_host_cap = 0;
  void* fetch_done = nullptr;  // cudaEvent_t: last descriptor upload finished reading fetch_host
  int64_t live_plans = 0;      // bat_plan_build plans not yet destroyed

  // pages released in stream order (bat_kv_release): reusable once `ev` has completed
  struct PendingFree {
    cudaEvent_t ev;
    std::vector<int32_t> pages;
  };
  std::deque<PendingFree> pending;
  std::vector<cudaEvent_t> spare_events;
  // double-buffered staging of pulled cold item pages for pre-built plans (bat_kv_staging_reserve)
  std::vector<std::vector<int32_t>> staging;

  const Entity* find(int32_t kind, int64_t id) const {
    auto it = index.find(EntityKey{kind, id});
    return it == index.end() ? nullptr : &it->second;
  }
  // Move pending pages back to the free list.  wait_stream != nullptr: make that stream wait for
  // their release events (no host blocking); otherwise the host waits for the events.
  bool reclaim(int64_t need, cudaStream_t wait_stream, bool use_stream) {
    while (static_cast<int64_t>(free_pages.size()) < need && !pending.empty()) {
      PendingFree& f = pending.front();
      cudaError_t e = use_stream ? cudaStreamWaitEvent(wait_stream, f.ev, 0) : cudaEventSynchronize(f.ev);
      if (e != cudaSuccess) return false;
      for (auto it = f.pages.rbegin(); it != f.pages.rend(); ++it) free_pages.push_back(*it);
      spare_events.push_back(f.ev);
      pending.pop_front();
    }
    return true;
  }
  // allocate n pages (all-or-nothing); pages still pending a stream-ordered release are reused
  // after a host wait on their release events (host-synchronous callers)
  bool alloc_pages(int64_t n, std::vector<int32_t>& out) {
    if (static_cast<int64_t>(free_pages.size()) < n) reclaim(n, nullptr, false);
    if (static_cast<int64_t>(free_pages.size()) < n) return false;
    for (int64_t i = 0; i < n; ++i) {
      out.push_back(free_pages.back());
      free_pages.pop_back();
    }
    return true;
  }
  // ... for asynchronous writers on `st`: pending pages are handed out behind a stream wait
  bool alloc_pages_on(int64_t n, std::vector<int32_t>& out, cudaStream_t st) {
    if (static_cast<int64_t>(free_pages.size()) < n) reclaim(n, st, true);
    if (static_cast<int64_t>(free_pages.size()) < n) return false;
    for (int64_t i = 0; i < n; ++i) {
      out.push_back(free_pages.back());
      free_pages.pop_back();
    }
    return true;
  }
  void release_pages(const std::vector<int32_t>& pages) {
    for (auto it = pages.rbegin(); it != pages.rend(); ++it) free_pages.push_back(*it);
  }
  int64_t n_free() const {
    int64_t n = static_cast<int64_t>(free_pages.size());
    for (const auto& f : pending) n += static_cast<int64_t>(f.pages.size());
    return n;
  }
};

// Cold items of a pre-built plan pulled into a staging slot (bat_plan_build_staged): the planner
// maps every remote (cold-sharded) prefix item to pages of the slot and records the copies.
struct StagingCtx {
  const std::vector<int32_t>* slot_pages = nullptr;
  size_t used = 0;
  std::unordered_map<EntityKey, Entity, EntityKeyHash> assigned;
  std::vector<uint64_t> src;  // peer-mapped source page addresses
  std::vector<int32_t> dst;   // local staging page ids
};

}  // namespace bat

// handle.cuh — the library handle (struct ggrid_s) and host helpers shared by api.cu and
// multi.cu.  Not part of the public ABI (include/ggrid.h).
#pragma once
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <utility>
#include <vector>

#include "ggrid.h"
#include "internal.cuh"

using namespace gg;

struct MultiIndex;  // multi.cu: a handle spanning several shards (devices or ranks)
struct Exchange;    // multi.cu: the transport between shards

namespace {  // (per translation unit)

bool debug_on() {
  static int v = -1;
  if (v < 0) v = getenv("GGRID_DEBUG") ? 1 : 0;
  return v == 1;
}

#define CK(x)                                                                             \
  do {                                                                                    \
    cudaError_t e_ = (x);                                                                 \
    if (e_ != cudaSuccess) {                                                              \
      if (debug_on()) fprintf(stderr, "ggrid: %s:%d %s: %s\n", __FILE__, __LINE__, #x,    \
                              cudaGetErrorString(e_));                                    \
      return e_ == cudaErrorMemoryAllocation ? GGRID_ENOMEM : GGRID_ECUDA;                \
    }                                                                                     \
  } while (0)

#define RC(x)                  \
  do {                         \
    int r_ = (x);              \
    if (r_ != GGRID_OK) return r_; \
  } while (0)

// grow-only device buffer
struct DBuf {
  void* p = nullptr;
  size_t n = 0;
  int ensure(size_t bytes) {
    if (bytes <= n) return GGRID_OK;
    if (p) cudaFree(p);
    p = nullptr;
    n = 0;
    size_t want = std::max<size_t>(bytes, 4096);
    if (cudaMalloc(&p, want) != cudaSuccess) {
      cudaGetLastError();
      return GGRID_ENOMEM;
    }
    n = want;
    return GGRID_OK;
  }
  void release() {
    if (p) cudaFree(p);
    p = nullptr;
    n = 0;
  }
  template <class T>
  T* as() const {
    return static_cast<T*>(p);
  }
};

bool is_device_ptr(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// pointer the kernels may dereference for p: p itself for device/managed memory, the mapped
// device alias for pinned host memory, null for pageable host memory (must be copied)
void* device_view(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) return const_cast<void*>(p);
  if (a.type == cudaMemoryTypeHost && a.devicePointer) {
    // offset of p inside its allocation maps 1:1 onto the device alias
    return static_cast<char*>(a.devicePointer) +
           (static_cast<const char*>(p) - static_cast<const char*>(a.hostPointer));
  }
  return nullptr;
}

}  // namespace

struct ggrid_s {
  int device = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  int sm_count = 148;
  uint32_t V = 0, A = 0, cs = 1, n_cells = 0, delta = 1, max_k = 256, max_objects = 0;
  int seed_neighbors = 1;
  uint32_t profile = 0;  // opts.profile: bit 0 = every kind, bit k+1 = kind k
  uint32_t t_delta = 0;  // message expiry window (0 = never)
  // asynchronous ingest (opts.async_ingest): ggrid_ingest returns once its kernels are queued.
  // Until the next sync the status mirror is stale by the batches queued since; these bound
  // what they can have added (records incl. extent padding, extents, newly live objects).
  int async_ingest = 0;
  int ingest_mode = 0;  // opts.ingest_kernels: 0 plan, 1 cell-hash launch, 2 direct launch, 3 three launches
  uint64_t pend_records = 0, pend_updates = 0;
  uint32_t pend_ext = 0;
  uint32_t max_cell_degree = 0;  // most neighbour cells of any cell
  std::vector<uint32_t> user_cell;
  DevGraph g{};
  DevState s{};
  std::vector<void*> allocs;
  DevStatus* d_status = nullptr;
  DevStatus* h_status = nullptr;  // pinned
  DevStatus* h_status_dev = nullptr;  // its mapped device alias (the kernels' store target)
  // Arrival order (reading R7): the key of an update is (t << 32) | seq with seq = seq_next + i.
  // seq starts at 1 (key 0 stays "no update"); when a batch would run past 2^32 - 1 the keys of
  // the whole index are re-based (rebase()), so a handle takes any number of updates.
  uint64_t seq_next = 1;
  uint64_t recs_since_flush = 0;  // records ingested since the last flush launch (kernel choice)
  int flush_kernel = 0;           // GGRID_FLUSH_KERNEL: 0 = by log length, 1 = ring, 2 = streaming, 3 = warp per cell
  uint64_t n_ingested = 0;  // updates accepted (or queued, asynchronous) so far
  uint64_t rebases = 0;
  uint32_t epoch = 0;
  DBuf upd_stage, tmp, q_stage, out_stage, lists, l2_scratch, dump_stage, gc_buf, misc, flush_spill,
      bound_stage, remote_stage, merge_stage;
  // pipelined ingest: two staging buffers filled on a copy stream
  struct Staged {
    DBuf buf;
    uint64_t n = 0;
    cudaEvent_t done = nullptr;      // copy finished (copy stream)
    cudaEvent_t consumed = nullptr;  // its ingest kernels finished reading it (main stream)
  };
  Staged staged[2];
  int stage_head = 0, n_staged = 0;
  Staged qstaged[2];  // staged query batches (ggrid_query_stage / ggrid_knn_commit)
  int qstage_head = 0, n_qstaged = 0;
  // multi-GPU (multi.cu): the front handle of an in-process index over several shards, or this
  // shard's transport when it is one rank of a multi-process index
  MultiIndex* multi = nullptr;
  Exchange* xchg = nullptr;
  DBuf mx[16];  // the exchange protocol's device buffers
  // prior-art query comparison path (prior_art_knn.cu): host copy of the out-arc CSR, made on
  // first use
  std::vector<uint32_t> pa_rowptr;
  std::vector<uint2> pa_adj;
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t ev_in = nullptr;   // caller's producer stream -> library streams (order_inputs)
  cudaEvent_t ev_out = nullptr;  // library stream -> a caller's stream (ggrid_signal_stream)
  DBuf chain_ring;
  DBuf resume_buf;  // resumable-promotion records (one per chain-ring slot, up to kResumeCap)
  DBuf qsort_buf;  // (GGRID_SORT_QUERIES experiment)  // queries promoted into the chained level (NONE = not yet written)
  ggrid_stats_t stats{};
  std::vector<std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>>> pending_ev;
  std::vector<cudaEvent_t> ev_pool;

  template <class T>
  int alloc(T** p, size_t count, bool zero = true) {
    *p = nullptr;
    size_t bytes = std::max<size_t>(count * sizeof(T), 16);
    if (cudaMalloc((void**)p, bytes) != cudaSuccess) {
      cudaGetLastError();
      return GGRID_ENOMEM;
    }
    allocs.push_back(*p);
    if (zero && cudaMemset(*p, 0, bytes) != cudaSuccess) return GGRID_ECUDA;
    return GGRID_OK;
  }

  cudaEvent_t get_event() {
    if (!ev_pool.empty()) {
      cudaEvent_t e = ev_pool.back();
      ev_pool.pop_back();
      return e;
    }
    cudaEvent_t e;
    cudaEventCreate(&e);
    return e;
  }

  // Order stream `on` after the work a caller queued on `producer` (cudaEventRecord +
  // cudaStreamWaitEvent: no host wait).  Caller memory a call reads (device updates, queries,
  // bounds) or writes (device / pinned outputs) may have been produced, or still be read, by
  // that work; without this the library's non-blocking stream could read a buffer before its
  // producer kernel wrote it (or overwrite it before the caller's reader ran).
  int order_after(cudaStream_t producer, cudaStream_t on) {
    if (producer == on) return GGRID_OK;
    CK(cudaEventRecord(ev_in, producer));
    CK(cudaStreamWaitEvent(on, ev_in, 0));
    return GGRID_OK;
  }
  // The default producer: the legacy default stream (whose operations wait for every blocking
  // stream) when the library runs on its own stream; the caller's own stream when opts.stream
  // was given (then the library's work is already in the caller's order).  Work on other
  // non-blocking streams is ordered with ggrid_wait_stream.
  int order_inputs(cudaStream_t on) { return order_after(own_stream ? cudaStreamLegacy : stream, on); }

  // every kernel launch goes through here: counted, and timed in profile mode
  template <class F>
  void launch(int kind, F&& f) {
    launch_on(kind, stream, f);
  }
  template <class F>
  void launch_on(int kind, cudaStream_t on, F&& f) {
    stats.launches++;
    stats.kernel_launches[kind]++;
    if (profile & (1u | (2u << kind))) {
      cudaEvent_t a = get_event(), b = get_event();
      cudaEventRecord(a, on);
      f();
      cudaEventRecord(b, on);
      pending_ev.push_back({kind, {a, b}});
    } else {
      f();
    }
  }

  // drain the stream, collect event timings, refresh the status mirror.  The mirror is written
  // by a kernel through its mapped alias, not a D2H cudaMemcpy: a copy would share the copy
  // engine with a staged ingest transfer and wait behind it.
  int sync() {
    launch(GGRID_K_OTHER, [&] { launch_copy_words(d_status, h_status_dev, sizeof(DevStatus), stream); });
    CK(cudaStreamSynchronize(stream));
    pend_records = pend_updates = 0;
    pend_ext = 0;
    for (auto& pe : pending_ev) {
      float ms = 0.f;
      if (cudaEventElapsedTime(&ms, pe.second.first, pe.second.second) == cudaSuccess)
        stats.kernel_ms[pe.first] += ms;
      ev_pool.push_back(pe.second.first);
      ev_pool.push_back(pe.second.second);
    }
    pending_ev.clear();
    CK(cudaGetLastError());
    return GGRID_OK;
  }

  // device-side word stores (a kernel: never queued behind a staged copy on a copy engine)
  int set_words(const WordSet& ws) {
    launch(GGRID_K_OTHER, [&] { launch_set_words(ws, stream); });
    return GGRID_OK;
  }
  int set_status_u32(unsigned int* field, unsigned int v) {
    WordSet ws;
    ws.add(field, v);
    return set_words(ws);
  }

  // fresh: st->flush_work and st->n_ovf were zeroed since the last flush (a knn's round 0)
  int flush_list_run(const Arena& out, unsigned long long* out_top, uint32_t begin, int full_vobj = 0,
                     uint32_t max_cells = 0, bool fresh = false) {
    const uint32_t opc = (uint32_t)((n_live_hi() + n_cells - 1) / std::max(1u, n_cells));
    uint32_t spill_cap = 0;
    const size_t sb = flush_spill_bytes(g.cs, opc, sm_count, &spill_cap);
    if (sb) RC(flush_spill.ensure(sb));
    uint32_t* spill = sb ? flush_spill.as<uint32_t>() : nullptr;
    // expiry (reading R21): drop extents whose newest t < t_now - t_delta
    const uint32_t t_now = h_status->t_max;
    const uint32_t t_cut = (t_delta && t_now > t_delta) ? t_now - t_delta : 0;
    // long cell logs (a bulk-ingested log, C1-size batches per cell) stream through the
    // bulk-copy ring; short ones (a few dozen records per cell per step) through the streaming
    // kernel, whose per-cell fixed cost is lower (C3 r2f: full flush 0.244 -> 0.224 ms with the
    // ring; the 1M-update step's flush 0.126 -> 0.155 ms with it)
    // (the warp-per-cell kernel for a step's short logs: one warp runs every phase of a cell, with
    // no CTA barrier; C3's 1M-update step flush 0.126 -> see DESIGN.md section 12)
    const uint64_t per_cell = recs_since_flush / std::max(1u, n_cells);
    int mode = FLUSH_STREAM;
    if (flush_kernel == 1 || (flush_kernel == 0 && per_cell >= 512)) mode = FLUSH_TMA;
    else if (!full_vobj && (flush_kernel == 3 || (flush_kernel == 0 && per_cell <= 128))) mode = FLUSH_WARP;
    if (mode == FLUSH_WARP && !fresh) {  // the warp kernel's cell counter and overflow list
      WordSet ws;
      ws.add(&d_status->flush_work, 0u);
      ws.add(&d_status->n_ovf, 0u);
      RC(set_words(ws));
    }
    launch(GGRID_K_FLUSH, [&] {
      launch_flush(g, s, out, out_top, begin, opc, full_vobj, sm_count, spill, spill_cap, t_cut, max_cells, mode,
                   stream);
    });
    if (mode == FLUSH_WARP)  // the cells with more extents or winners than a warp stages
      launch(GGRID_K_FLUSH, [&] {
        launch_flush(g, s, out, out_top, OVF_PASS, opc, 0, sm_count, spill, spill_cap, t_cut,
                     max_cells ? max_cells : (uint32_t)sm_count, FLUSH_STREAM, stream);
      });
    if (begin == 0) recs_since_flush = 0;
    return GGRID_OK;
  }

  int gc();
  int rebase();
  int ensure_arena(uint64_t need_records, uint32_t need_ext);
  // upper bound of the objects live on the device (exact after a sync)
  uint64_t n_live_hi() const {
    return std::min<uint64_t>(max_objects, (uint64_t)h_status->n_live + pend_updates);
  }
  // upper bound of the records a flush of every dirty cell can write: each live object is
  // valid in exactly one cell, plus <= 3 padding records per cell (dirty cells <= extents)
  uint64_t flush_need() const {
    return n_live_hi() + 4ull * std::min<uint64_t>(n_cells, (uint64_t)h_status->ext_top + pend_ext) + 16;
  }
  // the deferred error of an asynchronous ingest batch, as of the last sync (then cleared)
  int take_deferred() {
    const unsigned e = h_status->err_deferred | (async_ingest ? h_status->ingest_err : 0u);
    if (!e) return GGRID_OK;
    WordSet ws;
    ws.add(&d_status->err_deferred, 0u);
    ws.add(&d_status->ingest_err, 0u);
    RC(set_words(ws));
    h_status->err_deferred = 0;
    h_status->ingest_err = 0;
    return (e & (ERR_OBJ | ERR_EDGE | ERR_OFF)) ? GGRID_EINVAL : GGRID_ENOMEM;
  }
};


// api.cu: the single-shard paths the multi-shard driver (multi.cu) composes (defined inside
// api.cu's extern "C" block, hence the linkage; not exported through ggrid.h)
extern "C" {
__attribute__((visibility("hidden"))) int ingest_device(ggrid_t h, const uint4* d_u, uint64_t n);
__attribute__((visibility("hidden"))) int knn_impl(ggrid_t h, const ggrid_query* q, uint32_t n_q, uint32_t k, uint32_t* out_obj, uint32_t* out_dist,
             const uint32_t* bound = nullptr, uint64_t* out_remote = nullptr);
}
// multi.cu
int multi_build(const ggrid_graph* gr, uint32_t cell_size, const ggrid_opts& o, ggrid_t* out,
                int (*build_one)(const ggrid_graph*, uint32_t, const ggrid_opts&, ggrid_t*));
void multi_free(MultiIndex* mi);
const char* multi_exchange_name(const MultiIndex* mi);
uint32_t multi_n(const MultiIndex* mi);
ggrid_t multi_shard(const MultiIndex* mi, int r);
int multi_ingest(MultiIndex* mi, const ggrid_update* u, uint64_t n);
int multi_knn(MultiIndex* mi, const ggrid_query* q, uint32_t n_q, uint32_t k, uint32_t* out_obj, uint32_t* out_dist);
int rank_knn(ggrid_t h, const ggrid_query* q, uint32_t n_q, uint32_t k, uint32_t* out_obj, uint32_t* out_dist);
int rank_attach(ggrid_t h, const ggrid_opts& o);
void exchange_free(Exchange* e);
const char* exchange_name(const Exchange* e);

// internal.cuh — device-side data layout of the B200 G-Grid.
//
// Everything the hot path touches lives in HBM in flat arrays:
//   graph grid  : CSR over internal (Z-ordered) vertex ids; cells are runs of cell_size
//                 consecutive internal ids (P@11972-13692, reading R16), so cell(v) = v/cs.
//   object table: ot_key[o] = max (t<<32 | seq) over o's updates (P@15869, reading R7/R8).
//   message log : a bump-allocated record arena (SoA: obj, key, vsrc, off, edge) holding
//                 per-cell append-only extents (one per ingest batch per cell, a chain
//                 newest-first) = the paper's message lists of buckets (P@16303-17318),
//                 plus each cell's compacted object list (the cleaned result R[c],
//                 P@22008-22213) sorted by source vertex, indexed per vertex by v_obj.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "ggrid.h"

namespace gg {

constexpr uint32_t NONE = 0xFFFFFFFFu;
// cell_head[c] == STALE: no cached extents, but c's cleaned list holds a record of an object
// that has since reported from another cell (ingest marks it, reading R8); like a cell with
// cached updates it is re-cleaned before its list is read.  A chain ends at NONE or STALE.
constexpr uint32_t STALE = 0xFFFFFFFEu;
__host__ __device__ inline bool is_extent(uint32_t e) { return e < STALE; }
constexpr uint32_t INF = 0xFFFFFFFFu;  // u32 distance "unreachable" (reading R18)
constexpr unsigned long long EMPTY64 = ~0ull;
constexpr uint32_t BCOUNT_STRIDE = 32;
constexpr int EXPAND_LEVELS = 7;  // capacity ladder of the expansion (csrc/knn.cu)

enum ErrBits : unsigned {
  ERR_OBJ = 1u,      // update obj >= max_objects
  ERR_EDGE = 2u,     // update/query edge >= n_arcs
  ERR_OFF = 4u,      // offset >= w[edge]
  ERR_ARENA = 8u,    // arena / extent pool exhausted on device (should not happen)
  ERR_QUERY = 16u,   // query edge/offset invalid
  ERR_FAIL = 32u,    // a query overflowed the largest expansion variant
};

// Device-resident counters (one struct, read back with one D2H copy at sync points).
struct DevStatus {
  unsigned long long arena_top;  // next free record in the arena
  unsigned long long records_flushed;
  unsigned long long objects_written;
  unsigned long long cells_flushed;
  unsigned long long ex_iters, ex_vertices, ex_arcs, ex_harvested, ex_objects;  // expansion work
  unsigned long long records_expired;  // dropped unread by t_delta expiry
  unsigned long long ex_promoted, ex_retried;  // expansion outcomes: capacity overflow / dirty cell
  unsigned long long ex_resumed;  // promoted runs continued from their exported state
  unsigned int ext_top;     // next free extent
  unsigned int err;         // ErrBits of the current knn / flush / gc call
  unsigned int ingest_err;  // ErrBits of the current ingest batch (classify / alloc / scatter)
  unsigned int err_deferred;  // ingest_err of earlier asynchronous batches, not yet reported
  unsigned int bad_index;   // smallest offending index (ingest)
  unsigned int n_live;      // objects with at least one update
  unsigned int t_max;       // largest t ingested (t_now of the expiry rule)
  unsigned int n_flush;     // entries in flush_list
  unsigned int flush_work;  // persistent flush work counter
  unsigned int n_next[EXPAND_LEVELS];   // per expansion level: queries queued for the next round
  unsigned int flush_end;   // n_flush as seen by the last flush launch
  unsigned int expand_work[EXPAND_LEVELS];  // per-level dynamic work counters of the expand launches
  unsigned int n_chain;     // queries the starting level promoted into the chained level this round
  unsigned int l0_exited;   // CTAs of the starting level's launch that have exited this round
  unsigned int n_ovf;       // entries in ovf_list (this round's warp-per-cell flush)
  unsigned int round_end;   // (marks the end of the per-round reset region)
  unsigned int ingest_bar;  // grid-barrier arrivals of the fused ingest launch (reset per batch)
  unsigned int batch_tmax;  // newest t of the current ingest batch's valid updates (reset per
                            // batch); folded into t_max only once the batch is accepted
};

struct DevGraph {
  uint32_t V, A, cs, n_cells, delta;
  uint32_t cs_mul, cs_shift;  // v / cs by multiply-high (cs_mul = 0: cs is 2^cs_shift)
  const uint32_t* rowptr;    // [V+1] out-arc CSR by internal source
  const uint2* adj;          // [A]  (internal dst, w) in CSR order
  const uint2* einfo;        // [A]  user edge -> (internal src, w)
  const uint32_t* edst;      // [A]  user edge -> internal dst
  const uint32_t* cadj_ptr;  // [n_cells+1] cell adjacency (P@47172)
  const uint32_t* cadj;
  const uint2* vadj;         // [4V] inline adjacency: up to 4 (dst, w) per vertex; w=0 empty,
                             //      w=2^32-1: arcs 3.. of the vertex are in the CSR above
};

struct Arena {  // SoA record arena
  uint32_t* obj;
  unsigned long long* key;
  uint32_t* vsrc;
  uint32_t* off;
  uint32_t* edge;
  unsigned long long cap;
};

struct DevState {
  unsigned long long* ot_key;  // [max_objects]
  uint32_t max_objects;
  Arena ar;
  uint32_t* x_start;  // extents
  uint32_t* x_len;
  uint32_t* x_next;
  uint32_t* x_tmax;   // newest t of the extent's messages (zeta.t, P@20743)
  uint32_t ext_cap;
  uint32_t* cell_head;     // newest pending extent, or NONE (clean), or STALE (see above)
  uint32_t* listed_cell;   // [max_objects] the cell whose cleaned list holds o's record, or NONE
  uint32_t* cell_pending;  // cached records not yet cleaned
  uint32_t* cell_req;      // request epoch stamp (dedup of flush requests)
  uint2* v_obj;            // [V] (arena start, count) of the objects at each vertex
  uint32_t* vhas;          // [V/32 + 1] bit v: v may hold objects in its cell's cleaned list (a
                           // superset, rebuilt per cell by the flush): the query reads v_obj only
                           // for these (L2-resident: 3 MB at USA scale)
  uint2* cell_comp;        // [n_cells] (arena start, count) of the cell's compacted list
  uint32_t* vcnt;          // [V] flush scratch, only when cell_size > 4096 (else null)
  uint32_t* bcount;        // [n_cells * BCOUNT_STRIDE] per-batch count ([0]) and newest t ([1]),
                           // one 128-byte line per cell (same-line atomics from every ingest
                           // CTA serialise in L2)
  uint32_t* bbase;         // [n_cells] per-batch arena base
  uint32_t* flush_list;    // [n_cells]
  uint32_t* ovf_list;      // [n_cells] cells k_flush_warp left to the CTA kernel (st->n_ovf)
  DevStatus* st;
  // cell ownership across ranks: rank r owns the contiguous Z-order range of
  // cells c with floor(c * n_ranks / n_cells) == r; only owned cells keep logs and lists
  uint32_t n_ranks, rank;
};

__host__ __device__ inline uint32_t owner_of(uint32_t c, uint32_t n_cells, uint32_t n_ranks) {
  return (uint32_t)(((unsigned long long)c * n_ranks) / n_cells);
}

__host__ __device__ inline uint32_t cell_of(uint32_t v, uint32_t cs) { return v / cs; }

// cell(v) = v / cell_size without a hardware divide (Granlund-Montgomery round-up multiplier;
// exact for every 32-bit v, checked against v / d in tests/test_abi.py's reference of it)
inline void fastdiv_params(uint32_t d, uint32_t& mul, uint32_t& shift) {
  if ((d & (d - 1)) == 0) {
    mul = 0;
    shift = 0;
    while ((1u << shift) < d) ++shift;
    return;
  }
  uint32_t l = 0;
  while ((1ull << l) < d) ++l;  // ceil(log2 d)
  mul = (uint32_t)(((1ull << 32) * ((1ull << l) - d)) / d + 1);
  shift = l;
}
__device__ __forceinline__ uint32_t cellof(const DevGraph& g, uint32_t v) {
  if (g.cs_mul == 0) return v >> g.cs_shift;
  const uint32_t t = __umulhi(v, g.cs_mul);
  return (t + ((v - t) >> 1)) >> (g.cs_shift - 1);
}

// Programmatic dependent launch (the knn round's seed -> flush -> expansion chain): a kernel
// launched with pdl_config() may start while the previous one runs; it waits for it (and its
// memory) at pdl_wait() before touching anything, and lets its own dependent launch early with
// pdl_allow().  Both are no-ops for a normally launched kernel.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_allow() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
inline cudaLaunchConfig_t pdl_config(dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                                     cudaLaunchAttribute* attr) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cfg;
}

__device__ inline unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// Request a flush of cell c in this knn epoch (deduplicated by the epoch stamp).
// Ingest: an update of object o from cell c_new leaves o's record in the cleaned list of
// listed_cell[o] outdated when that is another cell: mark it STALE (unless it has cached
// extents already).  With this, a clean cell's list holds only latest records, so the query
// side needs no per-object validity gather (reading R8).
__device__ __forceinline__ void mark_moved(const DevState& s, uint32_t o, uint32_t c_new) {
  const uint32_t lc = s.listed_cell[o];
  if (lc != NONE && lc != c_new) atomicCAS(&s.cell_head[lc], NONE, STALE);
}

__device__ inline void request_flush(const DevState& s, uint32_t c, uint32_t epoch) {
  if (s.cell_head[c] == NONE) return;  // (clean; a STALE cell is re-cleaned too)
  // plain read first: most requests of a batch hit an already-requested cell, so the
  // contended atomic is only issued by the first few
  if (*((volatile uint32_t*)&s.cell_req[c]) == epoch) return;
  if (atomicExch(&s.cell_req[c], epoch) != epoch) {
    unsigned i = atomicAdd(&s.st->n_flush, 1u);
    s.flush_list[i] = c;
  }
}

}  // namespace gg

// Launchers (defined in the .cu files; called by api.cu).
namespace gg {
// A kernel attribute set once per (kernel, attribute, device): the attribute is a property of
// the kernel on the current device, so a process driving several devices needs it on each.
// Thread-safe; returns the cudaFuncSetAttribute result of the first call.
cudaError_t func_attr_once(const void* kernel, cudaFuncAttribute attr, int value);
template <class K>
inline cudaError_t func_attr_once(K* kernel, cudaFuncAttribute attr, int value) {
  return func_attr_once(reinterpret_cast<const void*>(kernel), attr, value);
}
// Small device-side word stores (status counters).  A kernel, not cudaMemset/cudaMemcpy: those
// can run on a copy engine and would queue behind a staged ingest transfer.
struct WordSet {
  static constexpr int N = 24;
  uint32_t* p[N];
  uint32_t v[N];
  int n = 0;
  // optional, applied before the stores: *fold_dst |= *fold_src (error bits carried over)
  uint32_t* fold_dst = nullptr;
  const uint32_t* fold_src = nullptr;
  void add(uint32_t* ptr, uint32_t val) {
    p[n] = ptr;
    v[n] = val;
    ++n;
  }
  void zero_range(uint32_t* ptr, int words) {
    for (int i = 0; i < words; ++i) add(ptr + i, 0u);
  }
};
void launch_set_words(const WordSet& ws, cudaStream_t st);
void launch_copy_words(const void* src, void* dst, size_t bytes, cudaStream_t st);
void launch_ingest_classify(const uint4* upd, uint64_t n, const DevGraph& g, const DevState& s,
                            uint2* tmp, cudaStream_t st);
// owner rank of each query's cell (cell of the query arc's source vertex)
void launch_query_owner(const uint2* q, uint32_t nq, const DevGraph& g, const DevState& s,
                        uint32_t* out_rank, cudaStream_t st);
// k-way merge of n_lists ascending (dist, obj) lists per query, layout [n_lists][n_q][k]
void launch_merge_topk(uint32_t n_lists, uint32_t n_q, uint32_t k, const uint32_t* lobj,
                       const uint32_t* ldist, uint32_t* out_obj, uint32_t* out_dist, cudaStream_t st);
size_t ingest_tmp_bytes(uint64_t n);
// single-launch ingest (classify + alloc + scatter with grid barriers) for batches that fit
// one resident wave; ingest_fused_plan returns false when the batch does not
struct IngestPlan {
  uint32_t grid, tile, ch;
  size_t smem;
  bool direct;  // k_ingest_direct (per-update rank atomics, registers across the barriers)
};
bool ingest_fused_plan(uint64_t n, uint32_t n_cells, int sm_count, int mode, IngestPlan* p);
// sort-by-cell ingest of a large batch (ingest_sort.cu): keys + radix sort + per-cell runs, then
// k_ingest_alloc, then the scatter of the sorted batch
struct SortedBatch {
  const uint32_t* keys;
  const unsigned long long* vals;
};
bool ingest_sorted_fits(uint64_t n);
size_t ingest_sort_tmp_bytes(uint64_t n, uint32_t n_cells);
cudaError_t launch_ingest_sorted_keys(const uint4* upd, uint64_t n, const DevGraph& g, const DevState& s,
                                      void* tmp, SortedBatch* out, cudaStream_t st);
void launch_ingest_sorted_scatter(const uint4* upd, uint64_t n, uint32_t seq0, const DevGraph& g,
                                  const DevState& s, const SortedBatch& b, cudaStream_t st);
cudaError_t launch_ingest_fused(const uint4* upd, uint64_t n, uint32_t seq0, const DevGraph& g,
                                const DevState& s, const IngestPlan& p, cudaStream_t st);  // classify -> scatter scratch (tmp + perm)
void launch_ingest_alloc(const DevGraph& g, const DevState& s, cudaStream_t st);
void launch_ingest_scatter(const uint4* upd, uint64_t n, uint32_t seq0, const DevGraph& g,
                           const DevState& s, const uint2* tmp, cudaStream_t st);
// q_copy (nullable): also store the queries there (q in mapped host memory)
enum SeedMode { SEED_DST = 0, SEED_NEIGHBORS = 1, SEED_ALL = 2 };
void launch_seed(const uint2* q, uint32_t nq, const DevGraph& g, const DevState& s, uint32_t epoch,
                 int mode, uint2* q_copy, cudaStream_t st);
// every nonzero key k of the arena's first n_records and of ot_key becomes (k & ~0xFFFFFFFF) | 1
void launch_rebase_keys(const DevState& s, unsigned long long n_records, cudaStream_t st);
void launch_mark_dirty(const DevGraph& g, const DevState& s, uint32_t epoch, int all_cells,
                       cudaStream_t st);
// Flush the cells flush_list[begin .. st->n_flush) writing compacted lists into `out`
// (out == s.ar for a regular flush; a fresh arena for garbage collection).
// spill: per-CTA global staging of winner positions beyond shared memory, sized by
// flush_spill_bytes (which also returns its per-buffer capacity; 0 = none needed)
size_t flush_spill_bytes(uint32_t cs, uint32_t objects_per_cell, int sm_count, uint32_t* cap);
// t_cut: extents whose newest t is below it are expired (dropped unread); 0 = none.
// max_ctas: an upper bound on the cells listed (0 = unknown): caps the persistent grid
// mode: FLUSH_STREAM the CTA-per-cell streaming kernel (k_flush), FLUSH_TMA its bulk-copy ring
// variant (k_flush_tma; long cell logs), FLUSH_WARP one warp per cell (k_flush_warp; short logs)
// followed by k_flush over the cells it could not take (s.ovf_list)
enum FlushMode { FLUSH_STREAM = 0, FLUSH_TMA = 1, FLUSH_WARP = 2 };
constexpr uint32_t OVF_PASS = 0xFFFFFFFFu;  // k_flush's `begin` for the overflow pass
void launch_flush(const DevGraph& g, const DevState& s, const Arena& out,
                  unsigned long long* out_top, uint32_t begin, uint32_t objects_per_cell,
                  int full_vobj, int sm_count, uint32_t* spill, uint32_t spill_cap, uint32_t t_cut,
                  uint32_t max_ctas, int mode, cudaStream_t st);

// v_obj[v] = (start, n) is valid only if start lies inside the cell's current cleaned list
// (lists only move up the arena between garbage collections, which rewrite every entry).
// (experiment hook) GG_VHAS=1: the flush maintains the may-hold-objects bitmap and the query reads a
// vertex's object index only when its bit is set.  Measured slower at C3 (r2i: expansion 1.367 ->
// 1.424 ms -- the index read becomes a second dependent trip for the vertices that hold objects --
// and the step's flush 0.127 -> 0.154 ms for the bitmap upkeep), so off: the index is read in the
// same round trip as the vertex's arcs.
#ifndef GG_VHAS
#define GG_VHAS 0
#endif
__device__ __forceinline__ bool vhas_bit(const DevState& s, uint32_t v) { return (s.vhas[v >> 5] >> (v & 31)) & 1u; }
__device__ __forceinline__ uint2 vobj_valid(uint2 vo, uint2 comp) {
  return (vo.x >= comp.x && vo.x < comp.x + comp.y) ? vo : make_uint2(0, 0);
}
// Expansion (Alg. 5/6 semantics) for the queries qlist[0..n) at variant `level`.
// Outcomes: answered (rows written), retried at the same level (retry_list, a needed cell
// had cached updates) or promoted to the next level (promote_list, capacity overflow).
// bound (nullable): per-query inclusive distance limit (objects farther are not returned and
// the search stops beyond it); remote (nullable): per-query bitmask of the ranks owning cells
// the search expanded into (sharded mode)
struct ExpandLaunch {
  int level = 0;
  const uint2* q = nullptr;
  const uint32_t* qlist = nullptr;  // (null: query i is qlist entry i)
  uint32_t n = 0;                   // queries in qlist
  uint32_t k = 0;
  uint32_t epoch = 0;
  uint32_t* retry_list = nullptr;   // this level, next round (counter: n_next[level])
  uint32_t* promote_list = nullptr; // next level
  uint32_t* promote_count = nullptr;
  uint32_t* out_obj = nullptr;
  uint32_t* out_dist = nullptr;
  const uint32_t* bound = nullptr;
  unsigned long long* remote = nullptr;
  void* scratch = nullptr;          // the last level's global working memory
  uint32_t scratch_warps = 0;
  // concurrency of a chained level with the level below it (same round, two streams):
  uint32_t* exited = nullptr;       // the lower level: each CTA counts itself out here
  const uint32_t* chain_in = nullptr;  // the chained level: queries promoted by the lower level,
                                       // appended after the n of qlist (entries NONE until written;
                                       // taken entries are reset to NONE)
  uint32_t chain_cap = 0;
  const uint32_t* wait_exited = nullptr;  // ... done when *wait_exited == wait_total
  uint32_t wait_total = 0;
  uint32_t grid = 0;                // 0: the default (expand_grid)
  bool trigger = false;             // let the next kernel of the stream start now (PDL)
  bool pdl = false;                 // launched as a programmatic dependent of the previous kernel
  uint32_t ball_hint = 0xFFFFFFFFu;  // expected ball (vertices): picks the starting level's variant
  // resumable promotions: records (expand_resume_bytes each) indexed by promotion-ring slot,
  // written by the one-warp starting level and read by the chained level (both get the buffer)
  void* resume = nullptr;
  uint32_t resume_cap = 0;
};
// CTAs launch_expand uses for n queries at `level` (ball_hint: expected ball in vertices)
uint32_t expand_grid(int level, uint32_t n, int sm_count, uint32_t ball_hint);
void launch_expand(const ExpandLaunch& L, const DevGraph& g, const DevState& s, int sm_count, cudaStream_t st);
// prior-art comparison path (csrc/prior_art.cu)
int prior_art_mu(int eta);
size_t prior_art_scan_bytes(uint32_t n);
size_t prior_art_bucket_bytes();
void launch_pa_count(const DevGraph& g, const DevState& s, uint32_t bsize, uint32_t* cnt, cudaStream_t st);
int launch_pa_scan(void* tmp, size_t tmp_bytes, const uint32_t* cnt, uint32_t* off, uint32_t n, cudaStream_t st);
void launch_pa_fill(const DevGraph& g, const DevState& s, uint32_t bsize, const uint32_t* off, void* out,
                    cudaStream_t st);
void launch_pa_shuffle(const DevState& s, const void* bk, uint32_t n_buckets, uint32_t bsize, int eta,
                       int write_mode, uint32_t n_bundles, void* T, cudaStream_t st);
void launch_pa_collect(const DevState& s, uint32_t max_objects, uint32_t n_bundles, const void* T,
                       uint32_t* out_edge, uint32_t* out_off, unsigned long long* counts, cudaStream_t st);
void launch_pa_bundle(const uint32_t* obj, const unsigned long long* key, int eta, uint32_t* out_obj,
                      unsigned long long* out_key, cudaStream_t st);
// queries ordered by their arcs' internal source vertex (cub radix sort): perm[i] = query index
size_t sort_queries_tmp_bytes(uint32_t n);
int launch_sort_queries(const uint2* q, uint32_t n, const DevGraph& g, void* tmp, size_t tmp_bytes, uint32_t* perm,
                        cudaStream_t st);
// shared memory of one CTA of a level's kernel in the mode a launch of n queries takes (chained:
// the level runs beside the one below it, CTA mode)
size_t expand_block_bytes(int level, uint32_t V, uint32_t n, int sm_count, uint32_t ball_hint, bool chained);
int expand_levels();
uint32_t expand_table_slots(int level);  // vertex-table capacity H of a level
uint32_t expand_max_k(int level);
size_t expand_warp_bytes(int level, uint32_t V);
// bytes per resumable-promotion record if `level` runs n queries one warp per query, else 0
size_t expand_resume_bytes(int level, uint32_t n, int sm_count, uint32_t ball_hint);
// the largest k the one-warp level-0 kernel takes, and the expected ball (vertices) from which the
// starting level runs one CTA per query: a larger k starts at the CTA kernel
uint32_t expand_warp_max_k();
uint32_t expand_cta_ball();
void launch_dump_cell(const DevGraph& g, const DevState& s, uint32_t c, uint32_t* obj,
                      uint32_t* edge, uint32_t* off, uint32_t cap, uint32_t* n_out, cudaStream_t st);
}  // namespace gg

// knn.cu — candidate construction and refinement of a kNN query (Alg. 4 lines 5-10,
// Alg. 5 GPU_SDist, GPU_First_k, Def. 3 GPU_Unresolved, Alg. 6 Refine_kNN;
// P@47779-52751), one warp per query.
//
// The paper runs |V| rounds of Bellman-Ford over the candidate cells with one thread per
// vertex (Alg. 5, P@48476-50421), picks the k nearest candidates, then refines them on CPU
// threads with one Dijkstra per unresolved boundary vertex (Alg. 6).  Both are prior art
// here.  This kernel computes the same exact answer with one bounded, label-correcting
// delta-stepping expansion per query that never leaves the GPU:
//
//   * D lives in a per-warp shared-memory open-addressing table keyed by vertex: a u32 key
//     array (a new vertex is claimed with a 32-bit atomicCAS) beside a u32 distance array
//     (relaxation = native 32-bit shared atomicMin, issued only when it improves; a 64-bit
//     (v<<32 | d) word would need a CAS loop: shared memory has no 64-bit min).  Seeds
//     follow reading R1 (d=0 -> D[src]=0, else D[dst]=w-d).
//   * Each round walks the frontier in chunks of 32; the vertices whose D lies in the bucket
//     [m, m+delta) (m = frontier minimum) are expanded 8 per window, lane = (vertex, slot):
//     each lane reads one arc of its vertex's 32-byte inline adjacency record (graph grid,
//     csrc/api.cu) — one dependent load per round, no degree scan.
//   * A vertex's objects are harvested the first time it is expanded (its cell's cleaned
//     list through the v_obj index, in the same memory round as its arcs) and kept as
//     (D-table slot, offset, object): a candidate's distance D[src(e_o)] + d_o (P@49436) is
//     re-read from the table when needed, so it is exact once the vertex is settled.
//     Objects on q's own arc ahead of q are at d_o - d_q (reading R2); stale entries are
//     dropped by key == ot_key.  Harvesting a vertex of a cell with cached updates requests
//     that cell's flush and the query is retried next round (lazy cleaning, Alg. 4 l.2-4).
//   * Stop once k candidates have dist < m (every object not yet harvested, or at an
//     unsettled vertex, is >= m): Def. 3's unresolved-vertex rule taken inclusively
//     (reading R13) and Alg. 6's refinement fused into the same expansion.  Output: the k
//     smallest (dist<<32 | obj) (readings R5, R6).
// Capacities are per variant ("level"); a query that overflows one is retried on the next.
#include <cstdio>
#include <algorithm>
#include <type_traits>

#include "internal.cuh"

namespace gg {

namespace {

enum { DONE = 0, RETRY = 1, OVERFLOW = 2 };
// (experiment hook) GG_TAIL_DEBUG=1: printf each level-0 promotion (reason, rounds, time) and each
// chained-level query's start/end times, to measure the promoted queries' tail
#ifndef GG_TAIL_DEBUG
#define GG_TAIL_DEBUG 0
#endif
__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#if GG_TAIL_DEBUG
#define OVF_AT(why) do { if (lane == 0) printf("P %u %d %u %u %llu\n", qi, (why), c_iter, nn, gtime()); return OVERFLOW; } while (0)
#else
#define OVF_AT(why) return OVERFLOW
#endif
// An overflow of the one-warp kernel inside a chunk (arc stage, table or frontier full) leaves a
// state the next level can resume from instead of restarting (see promote_export): the chunk's
// vertices harvested at this load lose their listed bits (their objects were not read yet) and
// the chunk and the rest of the bucket act[c0..na) stay to be expanded.
#define OVF_RES(why)                                                              \
  do {                                                                            \
    if (harv) atomicAnd(&m.listed[vslot >> 5], ~(1u << (vslot & 31)));             \
    rs.ok = true;                                                                 \
    rs.c0 = c0;                                                                   \
    rs.na = na;                                                                   \
    rs.nc = nc;                                                                   \
    rs.rmask = rmask;                                                             \
    __syncwarp();                                                                 \
    OVF_AT(why);                                                                  \
  } while (0)
#ifndef GG_MAXP
#define GG_MAXP 128
#endif
constexpr int MAXP = GG_MAXP;  // probe limit of the vertex table (slots)
constexpr uint32_t SPECIAL = 0xFFFFFFFFu;  // candidate slot of a same-arc object
constexpr uint32_t WMAX = 0xFFFFFFFFu;     // inline-adjacency overflow marker

// GG_BUCKET_HASH=1: the vertex table probes 4-slot buckets with one 16-byte load (a vertex is
// searched for in all four slots of a bucket at once; a new one claims the bucket's first free
// slot) instead of single slots -- fewer probe iterations, and so less lane divergence, at the
// same load.  C3 A/B: expansion 1.114 -> 1.054 ms (704 slots); 640 slots 1.076 (promotions)
#ifndef GG_BUCKET_HASH
#define GG_BUCKET_HASH 1
#endif
// GG_KD_INTERLEAVE=1: each 4-slot bucket keeps its 4 keys and then its 4 distances in one 32-byte
// block (one 16-byte load each, issued together), so a probe that finds its vertex already holds
// the vertex's distance; 0: separate key and distance arrays
// (measured at C3: 1.119 ms vs 1.046 ms separate -- the second 16-byte load and the lane
// selects cost more than the dependent distance load they save; off)
#ifndef GG_KD_INTERLEAVE
#define GG_KD_INTERLEAVE 0
#endif
static_assert(!GG_KD_INTERLEAVE || GG_BUCKET_HASH, "the interleaved table is a bucketed one");
constexpr uint32_t KB_STRIDE = GG_KD_INTERLEAVE ? 8u : 4u;  // words from one bucket's keys to the next's
#if GG_KD_INTERLEAVE
#define KEYR(M, I) ((M).key[(I) + ((I) & ~3u)])
#define DISTR(M, I) ((M).dist[(I) + ((I) & ~3u)])
#else
#define KEYR(M, I) ((M).key[(I)])
#define DISTR(M, I) ((M).dist[(I)])
#endif
#ifndef GG_BUCKET_ROT
#define GG_BUCKET_ROT 1  // (C3 A/B: 1.054 -> 1.046 ms)
#endif
struct Caps {
  uint32_t H, F, C;  // table slots, frontier, candidates
};

// byte layout of one query's working memory; S = the frontier's slot index type (u16 in shared
// memory, where tables have <= 16,384 slots; u32 for the global-memory level)
template <class S>
struct WarpMemT {
  uint32_t* key;             // H: vertex of the slot (EMPTY32 = free)
  uint32_t* dist;            // H: its tentative distance D
  unsigned long long* cand;  // C: (slot<<32 | offset); at the end (dist<<32 | obj)
  uint32_t* cobj;            // C: object ids
  S* front0;                 // F
  S* front1;                 // F
  uint32_t* fin;             // H/32: slot is in the frontier
  S* act;                    // F: the round's active slots (the bucket being expanded)
  uint32_t* listed;          // H/32 bits: vertex expanded at least once (objects harvested)
  uint2* stage;              // STAGE: the chunk's arcs (dst, D + w), compacted (one-warp variant)
};
using WarpMem = WarpMemT<uint32_t>;   // global-memory level
using WarpMemS = WarpMemT<uint16_t>;  // shared-memory levels
// arcs staged per chunk of 32 bucket vertices (at most 4 inline each = 128; a chunk with more real
// arcs than STAGE promotes its query -- rare: ~2.5 arcs per road vertex)
#ifndef GG_STAGE
#define GG_STAGE 112
#endif
constexpr uint32_t STAGE = GG_STAGE;
constexpr size_t STAGE_BYTES = 8ull * STAGE;
static_assert(STAGE >= 64, "a half chunk (16 vertices x 4 inline arcs) must fit the stage");
// a chunk with more arcs than the stage: staged in two halves (1) or its query promoted (0)
#ifndef GG_HALF_SPLIT
#define GG_HALF_SPLIT 0
#endif
// the chunk's harvest / rare-event vote after its relax passes (1) or before them (0)
#ifndef GG_LATE_EVENTS
#define GG_LATE_EVENTS 0  // (measured: 1.059 vs 1.046 ms -- off)
#endif

__host__ __device__ inline size_t warpmem_bytes(const Caps& c, size_t slot_bytes) {
  const size_t fr = (3ull * c.F * slot_bytes + 15) & ~size_t(15);
  return 8ull * c.C + STAGE_BYTES + 8ull * c.H + 4ull * c.C + 8ull * ((c.H + 31) / 32) + fr;
}

template <class S>
__device__ inline WarpMemT<S> carve(unsigned char* base, const Caps& c) {
  WarpMemT<S> m;
  m.cand = reinterpret_cast<unsigned long long*>(base);
  m.stage = reinterpret_cast<uint2*>(m.cand + c.C);
  uint32_t* p = reinterpret_cast<uint32_t*>(reinterpret_cast<unsigned char*>(m.stage) + STAGE_BYTES);
  m.key = p;
  m.dist = GG_KD_INTERLEAVE ? p + 4 : p + c.H;  // (interleaved: 4 keys, 4 distances per bucket)
  p += 2 * c.H;
  m.cobj = p; p += c.C;
  m.fin = p; p += (c.H + 31) / 32;
  m.listed = p; p += (c.H + 31) / 32;
  S* f = reinterpret_cast<S*>(p);
  m.front0 = f; f += c.F;
  m.front1 = f; f += c.F;
  m.act = f;
  return m;
}

// Fibonacci hashing (high bits, scaled to any table size H): ball vertex ids are Z-order
// clustered, so low-bit or identity hashing makes long probe runs
__device__ __forceinline__ uint32_t vhash(uint32_t v, uint32_t H) { return __umulhi(v * 2654435761u, H); }

constexpr uint32_t EMPTY32 = 0xFFFFFFFFu;  // free key slot (vertex ids are < 2^32-1)

// A vertex entering the frontier will be expanded in a later round: its inline adjacency record
// and object index are fetched into L2 now, so the expansion's dependent load hits L2 instead of
// DRAM (the USA-shaped graph's 0.9 GB of per-vertex records is far beyond L2).
#ifndef GG_PREFETCH_VOBJ
#define GG_PREFETCH_VOBJ 1
#endif
#ifndef GG_PREFETCH
#define GG_PREFETCH 1  // (C3: expansion 1.75 -> 1.66 ms per 65,536 queries, r2b variants)
#endif
// (experiment hook) issue the first chunk's loads before the termination count: measured no
// different at C3 (1.277 vs 1.280 ms, r2p) at 72 instead of 56 registers -- off
#ifndef GG_EARLY_LOADS
#define GG_EARLY_LOADS 0
#endif
// one-warp variant: lane = vertex chunks with compacted arcs (1) or lane = (vertex, slot)
// windows of 8 vertices (0, the round-1 design)
#ifndef GG_WARP_ARCS
#define GG_WARP_ARCS 1
#endif
// the final candidate sort in registers (shuffles) when at most 32 candidates and k <= 32 (1)
#ifndef GG_REG_SORT
#define GG_REG_SORT 1
#endif
// the one-warp table cleared with 16-byte stores (1) or 4-byte ones (0)
#ifndef GG_VEC_INIT
#define GG_VEC_INIT 1
#endif
static_assert(INF == EMPTY32, "a cleared slot's key and distance are the same word");
__device__ __forceinline__ void prefetch_vertex(const DevGraph& g, const DevState& s, uint32_t v) {
  if (GG_PREFETCH) {
    asm volatile("prefetch.global.L2 [%0];" ::"l"(g.vadj + (size_t)v * 4));
    if (!GG_VHAS && GG_PREFETCH_VOBJ) asm volatile("prefetch.global.L2 [%0];" ::"l"(s.v_obj + v));
  }
}

// A record read from a clean cell's list is its object's latest (ingest marks a cell whose list
// an object has left STALE, and the query re-cleans STALE cells like dirty ones: reading R8), so
// the object-table gather key == ot_key[obj] is only a debug cross-check (GG_HARVEST_VALIDATE=1).
#ifndef GG_HARVEST_VALIDATE
#define GG_HARVEST_VALIDATE 0
#endif
__device__ __forceinline__ bool valid_rec(const DevState& s, uint32_t p, uint32_t ob) {
  return !GG_HARVEST_VALIDATE || s.ar.key[p] == s.ot_key[ob];
}

template <class M>
__device__ __forceinline__ uint4 ld_words4(const M& m, const uint32_t* p) {
  uint4 r;
  if constexpr (sizeof(*m.front0) == 2) {  // (shared-memory levels)
    const uint32_t a = (uint32_t)__cvta_generic_to_shared(p);
    asm volatile("ld.volatile.shared.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "r"(a));
  } else {
    asm volatile("ld.volatile.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  }
  return r;
}
template <class M>
__device__ __forceinline__ uint4 ld_bucket(const M& m, uint32_t b) { return ld_words4(m, m.key + KB_STRIDE * b); }
// the slot of v in bucket b's keys kk, or -1
__device__ __forceinline__ int bucket_match(const uint4& kk, uint32_t b, uint32_t v) {
  const uint32_t mm = (kk.x == v ? 1u : 0u) | (kk.y == v ? 2u : 0u) | (kk.z == v ? 4u : 0u) | (kk.w == v ? 8u : 0u);
  return mm ? (int)(4 * b + __ffs(mm) - 1) : -1;
}

// insert-or-min of (v, d); returns the slot (or -1 if the table is full)
template <class M>
__device__ __forceinline__ int tab_relax(const M& m, uint32_t H, uint32_t v, uint32_t d,
                                         bool& improved) {
#if GG_BUCKET_HASH
  // buckets b, b+1, ... (linear probing over buckets): v is in the first bucket holding it or a
  // free slot (slots are never freed, so a bucket with a free slot ends every search)
  const uint32_t NB = H >> 2;
  uint32_t b = vhash(v, NB);
  int fs = -1;
  uint32_t dpre = INF;  // (interleaved table) the slot's distance as loaded with its bucket
#pragma unroll 1
  for (int p = 0; p < MAXP / 4 && fs < 0; ++p) {
    uint4 kk = ld_bucket(m, b);
    uint4 dd = make_uint4(INF, INF, INF, INF);
    if (GG_KD_INTERLEAVE) dd = ld_words4(m, m.key + KB_STRIDE * b + 4);
#pragma unroll 1
    for (;;) {
      fs = bucket_match(kk, b, v);
      if (fs >= 0) {
        const uint32_t jj = (uint32_t)fs & 3u;
        dpre = jj == 0 ? dd.x : jj == 1 ? dd.y : jj == 2 ? dd.z : dd.w;
        break;
      }
      const uint32_t e = (kk.x == EMPTY32 ? 1u : 0u) | (kk.y == EMPTY32 ? 2u : 0u) |
                         (kk.z == EMPTY32 ? 4u : 0u) | (kk.w == EMPTY32 ? 8u : 0u);
      if (!e) break;  // full: the next bucket
#if GG_BUCKET_ROT
      // the first free slot at or after slot (v & 3) (cyclically): lanes claiming different
      // vertices in one bucket mostly aim at different slots (fewer failed CAS rounds)
      const uint32_t r = v & 3u, e2 = e | (e << 4);
      const uint32_t j = 4 * b + ((__ffs(e2 >> r) - 1 + r) & 3u);
#else
      const uint32_t j = 4 * b + __ffs(e) - 1;
#endif
      const uint32_t old = atomicCAS(&KEYR(m, j), EMPTY32, v);
      if (old == EMPTY32 || old == v) {
        fs = (int)j;
        dpre = INF;  // (just claimed: the atomicMin below decides)
        break;
      }
      kk = ld_bucket(m, b);  // another lane took that slot: look again
    }
    b = b + 1 == NB ? 0 : b + 1;
  }
  if (fs < 0) {
    improved = false;
    return -1;
  }
  const uint32_t sl = (uint32_t)fs;
  // (a stale preloaded distance is never below the current one: distances only decrease)
  const uint32_t dnow = GG_KD_INTERLEAVE ? dpre : *(volatile uint32_t*)&DISTR(m, sl);
#else
  uint32_t sl = vhash(v, H);
  // find or claim v's slot (one exit; the distance update below is out of the probe loop)
#pragma unroll 1
  for (int p = 0;; ++p) {
    uint32_t cur = *(volatile uint32_t*)&KEYR(m, sl);
    if (cur == EMPTY32) {
      cur = atomicCAS(&KEYR(m, sl), EMPTY32, v);
      if (cur == EMPTY32) cur = v;  // claimed (its distance is still INF)
    }
    if (cur == v) break;
    if (p + 1 == MAXP) {
      improved = false;
      return -1;
    }
    sl = sl + 1 == H ? 0 : sl + 1;
  }
#endif
#if !GG_BUCKET_HASH
  const uint32_t dnow = *(volatile uint32_t*)&DISTR(m, sl);
#endif
  if (dnow <= d) {  // not an improvement (e.g. the twin arc back)
    improved = false;
  } else {
    improved = atomicMin(&DISTR(m, sl), d) > d;
  }
  return (int)sl;
}

// warp bitonic sort of a[0..n) ascending (n padded to a power of two <= cap)
__device__ void warp_sort(unsigned long long* a, uint32_t n, uint32_t cap, int lane) {
  uint32_t n2 = 1;
  while (n2 < n) n2 <<= 1;
  if (n2 > cap) n2 = cap;
  for (uint32_t i = n + lane; i < n2; i += 32) a[i] = EMPTY64;
  __syncwarp();
  for (uint32_t size = 2; size <= n2; size <<= 1) {
    for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
      for (uint32_t i = lane; i < n2 / 2; i += 32) {
        const uint32_t lo = 2 * i - (i & (stride - 1));
        const uint32_t hi = lo + stride;
        const bool asc = (lo & size) == 0;
        const unsigned long long x = a[lo], y = a[hi];
        if ((x > y) == asc) {
          a[lo] = y;
          a[hi] = x;
        }
      }
      __syncwarp();
    }
  }
}

// State of a query promoted out of the one-warp kernel mid-search (OVF_RES), resumed by the
// chained level instead of restarted: at C3 the promoted queries (~28 of 65,536, all on a full
// 704-slot table) overflow after ~90% of their rounds, and a restart at the next level put
// ~100 us of serial search after the starting level's end.
struct Resume {
  bool ok;
  uint32_t c0, na, nc;
  unsigned long long rmask;
};
// record layout (global memory, one per promotion-ring slot; caps = the exporting level's):
// header {qi, n_act, nc, valid, rmask}, key[H], dist[H], listed[W], fin[W], act[F], cand[C],
// cobj[C]  (W = H/32 words; the slots of act/cand refer to the exported table)
struct RecHdr {
  uint32_t qi, n_act, nc, valid;
  unsigned long long rmask;
  uint32_t pad[2];
};
static_assert(sizeof(RecHdr) == 32, "resume record header");
struct RecView {
  RecHdr* hdr;
  uint32_t *key, *dist, *listed, *fin, *act;
  unsigned long long* cand;
  uint32_t* cobj;
};
__host__ __device__ inline size_t resume_bytes(const Caps& c) {
  const size_t w = (c.H + 31) / 32;
  return (sizeof(RecHdr) + 8ull * c.H + 8ull * w + 4ull * (c.F + (c.F & 1u)) + 12ull * c.C + 15) & ~size_t(15);
}
__device__ inline RecView rec_view(unsigned char* base, const Caps& c) {
  RecView r;
  const uint32_t w = (c.H + 31) / 32;
  r.hdr = reinterpret_cast<RecHdr*>(base);
  r.key = reinterpret_cast<uint32_t*>(base + sizeof(RecHdr));
  r.dist = r.key + c.H;
  r.listed = r.dist + c.H;
  r.fin = r.listed + w;
  r.act = r.fin + w;
  r.cand = reinterpret_cast<unsigned long long*>(r.act + c.F + (c.F & 1u));  // (8-byte aligned)
  r.cobj = reinterpret_cast<uint32_t*>(r.cand + c.C);
  return r;
}

// slot of a vertex known to be in the table (-1: not found)
template <class M>
__device__ __forceinline__ int tab_find(const M& m, uint32_t H, uint32_t v) {
#if GG_BUCKET_HASH
  const uint32_t NB = H >> 2;
  uint32_t b = vhash(v, NB);
  for (int p = 0; p < MAXP / 4; ++p) {
    const uint4 kk = ld_bucket(m, b);
    const int sl = bucket_match(kk, b, v);
    if (sl >= 0) return sl;
    b = b + 1 == NB ? 0 : b + 1;
  }
  return -1;
#endif
  uint32_t sl = vhash(v, H);
  for (int p = 0; p < MAXP; ++p) {
    if (KEYR(m, sl) == v) return (int)sl;
    sl = sl + 1 == H ? 0 : sl + 1;
  }
  return -1;
}

struct QParams {
  DevGraph g;
  DevState s;
  const uint2* q;
  const uint32_t* qlist;
  uint32_t n;
  uint32_t k;
  uint32_t epoch;
  int level;
  int last_level;
  uint32_t* retry_list;     // same level, next round
  uint32_t* promote_list;   // next level (this round when chained, else the next round)
  uint32_t* promote_count;  // its counter
  uint32_t* out_obj;
  uint32_t* out_dist;
  const uint32_t* bound;          // per-query inclusive distance limit, or null
  unsigned long long* remote;     // per-query mask of other ranks' cells reached, or null
  Caps caps;
  unsigned char* scratch;   // global working memory (last level) or null (shared)
  uint32_t warps_per_cta;
  uint32_t* exited;               // (see ExpandLaunch)
  uint32_t* chain_in;
  uint32_t chain_cap;
  const uint32_t* wait_exited;
  uint32_t wait_total;
  int trigger;
  int wait_prior;  // launched as a programmatic dependent that must see the previous grid (flush)
  // resumable promotions (one-warp starting level -> chained level): one record per ring slot
  unsigned char* resume;
  uint32_t resume_cap;    // records (ring slots at or past it promote without state)
  uint32_t resume_bytes;  // bytes per record
  Caps rcaps;             // the exporting level's capacities (record layout)
};

// programmatic dependent launch: the next kernel of the stream may start right away (it
// depends on this one only through the promotion ring and the exit counter)
__device__ __forceinline__ void pdl_trigger(const QParams& P) {
  if (P.wait_prior) pdl_wait();  // the round's flush has finished and its lists are visible
  if (P.trigger) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

// a CTA of a lower level leaving: publishes its promotions to a concurrent chained level
__device__ __forceinline__ void count_exit(const QParams& P) {
  if (P.exited) {
    __threadfence();
    const uint32_t o = atomicAdd(P.exited, 1u);
#if GG_TAIL_DEBUG
    if (o + 1 == gridDim.x) printf("E %llu\n", gtime());
#else
    (void)o;
#endif
  }
}

// current distance of candidate i (exact once its source vertex is settled)
template <class M>
__device__ __forceinline__ unsigned long long cand_dist(const M& m, uint32_t i) {
  const unsigned long long a = m.cand[i];
  const uint32_t slot = (uint32_t)(a >> 32), off = (uint32_t)a;
  if (slot == SPECIAL) return off;
  return (unsigned long long)DISTR(m, slot) + off;
}

// Append one ballot's worth of candidates (false: capacity exceeded)
template <class M>
__device__ __forceinline__ bool cand_push(const M& m, uint32_t& nc, uint32_t C, bool has,
                                          uint32_t slot, uint32_t off, uint32_t obj, unsigned lt) {
  const unsigned hm = __ballot_sync(0xffffffffu, has);
  if (!hm) return true;
  if (nc + __popc(hm) > C) return false;
  if (has) {
    const uint32_t i = nc + __popc(hm & lt);
    m.cand[i] = ((unsigned long long)slot << 32) | off;
    m.cobj[i] = obj;
  }
  nc += __popc(hm);
  return true;
}

// Ask for the flush of every dirty cell the frontier will need, so a retried query is
// unlikely to stop again for the same reason.
template <class M, class S>
__device__ void request_lookahead(const QParams& P, const M& m, const S* front, uint32_t nf, int lane) {
  for (uint32_t i = lane; i < nf; i += 32) {
    const uint32_t v = KEYR(m, front[i]);
    request_flush(P.s, cellof(P.g, v), P.epoch);
  }
}

// a query not answered at this level: retried here next round (a needed cell had cached
// updates), or promoted to the next level (capacity overflow)
__device__ void finish_undone(const QParams& P, uint32_t qi, int r) {
  if (r == RETRY) {
    atomicAdd(&P.s.st->ex_retried, 1ull);
    P.retry_list[atomicAdd(&P.s.st->n_next[P.level], 1u)] = qi;
  } else if (P.level < P.last_level) {
    atomicAdd(&P.s.st->ex_promoted, 1ull);
    P.promote_list[atomicAdd(P.promote_count, 1u)] = qi;
#if GG_TAIL_DEBUG
    printf("Q %u %llu\n", qi, gtime());
#endif
  } else {
    atomicOr(&P.s.st->err, (unsigned)ERR_FAIL);
  }
}

// Promotion of a query that overflowed the one-warp kernel, to the chained level: the ring slot
// is taken first, the working state (OVF_RES) is written to that slot's record, then the ring
// entry is published (fence: a reader that sees the entry sees the record).  A state that cannot
// be resumed (rs.ok false) is published with valid = 0 and the next level restarts the query.
template <class M>
__device__ void promote_export(const QParams& P, const M& m, uint32_t qi, int lane, const Resume& rs) {
  uint32_t t = 0;
  if (lane == 0) {
    atomicAdd(&P.s.st->ex_promoted, 1ull);
    t = atomicAdd(P.promote_count, 1u);
  }
  t = __shfl_sync(0xffffffffu, t, 0);
  if (t < P.resume_cap) {
    const Caps& c = P.caps;
    const RecView r = rec_view(P.resume + (size_t)t * P.resume_bytes, c);
    const uint32_t n_act = rs.ok ? rs.na - rs.c0 : 0;
    if (rs.ok) {
      for (uint32_t i = lane; i < c.H; i += 32) {
        r.key[i] = KEYR(m, i);
        r.dist[i] = DISTR(m, i);
      }
      for (uint32_t i = lane; i < (c.H + 31) / 32; i += 32) {
        r.listed[i] = m.listed[i];
        r.fin[i] = m.fin[i];
      }
      for (uint32_t i = lane; i < n_act; i += 32) r.act[i] = m.act[rs.c0 + i];
      for (uint32_t i = lane; i < rs.nc; i += 32) {
        r.cand[i] = m.cand[i];
        r.cobj[i] = m.cobj[i];
      }
    }
    if (lane == 0) {
      RecHdr h;
      h.qi = qi;
      h.n_act = n_act;
      h.nc = rs.ok ? rs.nc : 0;
      h.valid = rs.ok ? 1u : 0u;
      h.rmask = rs.rmask;
      h.pad[0] = h.pad[1] = 0;
      *r.hdr = h;
    }
    __threadfence();
  }
  __syncwarp();
#if GG_TAIL_DEBUG
  if (lane == 0) printf("Q %u %llu\n", qi, gtime());
#endif
  if (lane == 0) P.promote_list[t] = qi;
}

template <class M>
__device__ __forceinline__ int run_query(const QParams& P, const M& m, uint32_t qi, int lane, Resume& rs) {
  const unsigned FULL = 0xffffffffu;
  const DevGraph& g = P.g;
  const DevState& s = P.s;
  const Caps& cp = P.caps;
  const uint32_t H = cp.H;
  const uint32_t k = P.k;
  const unsigned lt = lanemask_lt();

  if (GG_VEC_INIT && (cp.H & 3u) == 0) {  // 16-byte stores (carve() keeps both arrays 16-aligned)
    const uint4 e4 = make_uint4(EMPTY32, EMPTY32, EMPTY32, EMPTY32);
    if (GG_KD_INTERLEAVE) {  // (keys and distances: one 2H-word block)
      for (uint32_t i = lane; i < cp.H / 2; i += 32) reinterpret_cast<uint4*>(m.key)[i] = e4;
    } else {
      for (uint32_t i = lane; i < cp.H / 4; i += 32) {
        reinterpret_cast<uint4*>(m.key)[i] = e4;
        reinterpret_cast<uint4*>(m.dist)[i] = e4;  // (INF == EMPTY32)
      }
    }
  } else {
    for (uint32_t i = lane; i < cp.H; i += 32) {
      KEYR(m, i) = EMPTY32;
      DISTR(m, i) = INF;
    }
  }
  for (uint32_t i = lane; i < (cp.H + 31) / 32; i += 32) m.fin[i] = 0;
  for (uint32_t i = lane; i < (cp.H + 31) / 32; i += 32) m.listed[i] = 0;
  __syncwarp();

  const uint2 q = P.q[qi];
  if (q.x >= g.A) return DONE;   // invalid query: reported by the seed kernel (EINVAL)
  const uint2 ei = g.einfo[q.x];  // (internal src, w)
  if (q.y >= ei.y) return DONE;
  // sharded mode: objects only from this rank's cells; the owners of other cells the search
  // expands into are collected (they are asked for their objects within the final radius)
  const uint32_t lim = P.bound ? P.bound[qi] : INF;
  const bool track = P.remote != nullptr && s.n_ranks > 1;
  unsigned long long rmask = 0;
  if (track) {
    const uint32_t o = owner_of(cellof(g, ei.x), g.n_cells, s.n_ranks);
    if (o != s.rank) rmask |= 1ull << o;  // same-arc objects ahead of q live at src(q.e)
  }
  uint32_t seed_v, seed_d;
  if (q.y == 0) {
    seed_v = ei.x;
    seed_d = 0;
  } else {
    seed_v = g.edst[q.x];
    seed_d = ei.y - q.y;
  }
  auto* front = m.front0;
  auto* nfront = m.front1;
  uint32_t nf = 1, nc = 0;
  if (lane == 0) {
    bool imp;
    const int sl = tab_relax(m, H, seed_v, seed_d, imp);
    front[0] = (uint32_t)sl;
    m.fin[sl >> 5] |= 1u << (sl & 31);
  }
  __syncwarp();

  // objects on q's own arc ahead of q (reading R2); they are stored at vertex src(q.e)
  if (q.y > 0) {
    const uint32_t c = cellof(g, ei.x);
    if (s.cell_head[c] != NONE) {
      if (lane == 0) request_flush(s, c, P.epoch);
      return RETRY;
    }
    const uint2 vo = vobj_valid(s.v_obj[ei.x], s.cell_comp[c]);
    for (uint32_t j0 = 0; j0 < vo.y; j0 += 32) {
      const uint32_t j = j0 + lane;
      bool has = false;
      uint32_t ob = 0, dd = 0;
      if (j < vo.y) {
        const uint32_t p = vo.x + j;
        ob = s.ar.obj[p];
        const uint32_t oe = s.ar.edge[p], oo = s.ar.off[p];
        if (oe == q.x && oo >= q.y && valid_rec(s, p, ob)) {
          has = true;
          dd = oo - q.y;
        }
      }
      if (!cand_push(m, nc, cp.C, has, SPECIAL, dd, ob, lt)) return OVERFLOW;
    }
    __syncwarp();
  }

  // work counters: c_iter / c_vert warp-uniform, the others per lane (reduced at the end)
  uint32_t c_iter = 0, c_vert = 0, c_arcs = 0, c_harv = 0, c_objs = 0;
  // frontier minimum, maintained across rounds: the next frontier holds the re-queued
  // entries (their D read at partition) and every vertex improved during the round (each
  // improvement's new D is seen here), so min over those is exact
  uint32_t blo = seed_d;
  struct Win {
    uint32_t vslot, u, hcell, hd;
    uint2 arc, cc, v0;
    bool vv, harv;
  };
  for (;;) {
    ++c_iter;
    // ---- 1. termination: k candidates strictly closer than anything not yet final ---------
    if (nf == 0) break;
    if (blo > lim) break;  // every object not yet harvested is beyond the caller's bound
    auto terminated = [&]() {
      if (nc < k) return false;
      uint32_t cl = 0;
      for (uint32_t i = lane; i < nc; i += 32) cl += cand_dist(m, i) < blo;
      return __reduce_add_sync(FULL, cl) >= k;
    };
    if ((!GG_EARLY_LOADS || !GG_WARP_ARCS) && terminated()) break;

    // ---- 2. partition the frontier: the bucket [m, m + delta) into act, the rest re-queued --
    const uint32_t bhi = (blo > INF - g.delta) ? INF : blo + g.delta;
    uint32_t nn = 0, na = 0, mn = INF;
    for (uint32_t b0 = 0; b0 < nf; b0 += 32) {
      const uint32_t i = b0 + lane;
      const uint32_t sl = i < nf ? front[i] : NONE;
      const uint32_t ent = sl != NONE ? DISTR(m, sl) : INF;
      const bool a = sl != NONE && ent < bhi;
      const bool r = sl != NONE && !a;
      const unsigned rm = __ballot_sync(FULL, r);
      if (r) {
        nfront[nn + __popc(rm & lt)] = sl;
        mn = min(mn, ent);
      }
      nn += __popc(rm);
      const unsigned am = __ballot_sync(FULL, a);
      if (a) {
        m.act[na + __popc(am & lt)] = sl;
        atomicAnd(&m.fin[sl >> 5], ~(1u << (sl & 31)));  // re-queued if improved from here on
      }
      na += __popc(am);
    }
    __syncwarp();
    if (!GG_EARLY_LOADS || !GG_WARP_ARCS) c_vert += na;

#if GG_WARP_ARCS
    // ---- 3. expand the bucket in chunks of 32 vertices, lane = vertex: ONE dependent global
    //         round trip per chunk loads each vertex's 32-byte inline arc record (two 16-byte
    //         loads) and, at its first expansion, its cell state and object index; the chunk's
    //         real arcs are then compacted into shared memory (warp prefix sum over the lanes'
    //         arc counts) and relaxed 32 at a time, lane = arc -- no lane idles on an empty slot
    struct ChunkLd {
      uint32_t vslot, u, du, hcell, hd;
      uint4 a01, a23;
      uint2 cc, v0;
      bool vv, harv;
    };
    auto load_chunk = [&](uint32_t c0) {
      ChunkLd x;
      const uint32_t vi = c0 + lane;
      x.vv = vi < na;
      x.vslot = 0;
      x.u = 0;
      x.du = INF;
      x.hcell = 0;
      x.hd = NONE;
      x.a01 = make_uint4(0, 0, 0, 0);
      x.a23 = make_uint4(0, 0, 0, 0);
      x.cc = make_uint2(0, 0);
      x.v0 = make_uint2(0, 0);
      x.harv = false;
      if (x.vv) {
        x.vslot = m.act[vi];
        x.u = KEYR(m, x.vslot);
        x.du = DISTR(m, x.vslot);  // (an improvement after this read re-queues the vertex: fin cleared)
        const uint4* rec = reinterpret_cast<const uint4*>(g.vadj + (size_t)x.u * 4);
        x.a01 = rec[0];
        x.a23 = rec[1];
        x.harv = !(atomicOr(&m.listed[x.vslot >> 5], 1u << (x.vslot & 31)) & (1u << (x.vslot & 31)));
        if (x.harv) {
          x.hcell = cellof(g, x.u);
          x.hd = s.cell_head[x.hcell];
          x.cc = s.cell_comp[x.hcell];
          if (!GG_VHAS || vhas_bit(s, x.u)) x.v0 = s.v_obj[x.u];  // (GG_VHAS: most hold no object)
        }
      }
      return x;
    };
    // (GG_EARLY_LOADS) the first chunk's global loads go out before the termination count, whose
    // shared-memory work then overlaps their latency; a stopping round just drops them
    ChunkLd first;
    if (GG_EARLY_LOADS) {
      first = load_chunk(0);
      if (terminated()) break;
      c_vert += na;  // (counted for expanded rounds only)
    }
    for (uint32_t c0 = 0; c0 < na; c0 += 32) {
      const ChunkLd x = (GG_EARLY_LOADS && c0 == 0) ? first : load_chunk(c0);
      const uint32_t vslot = x.vslot, u = x.u, du = x.du, hcell = x.hcell, hd = x.hd;
      const uint4 a01 = x.a01, a23 = x.a23;
      const uint2 cc = x.cc, v0 = x.v0;
      const bool harv = x.harv;
      const bool overflow_arcs = a23.w == WMAX;  // more than 4 arcs: 3 inline, the rest in the CSR
      // compact the real arcs (w != 0) of the chunk: (dst, du + w), skipping sums >= INF
      // a real arc (1 <= w < WMAX) whose sum stays below INF (du < INF: a bucket vertex); 32-bit
      const uint32_t room = INF - du;
      auto real = [&](uint32_t w) { return (w - 1u < WMAX - 1u) & (w < room); };
      const uint32_t r0 = real(a01.y), r1 = real(a01.w), r2 = real(a23.y), r3 = real(a23.w);
#if !GG_LATE_EVENTS
      const bool dirty = harv && hd != NONE;
      const uint2 vo = harv ? vobj_valid(v0, cc) : make_uint2(0, 0);
      const uint32_t ev = __reduce_or_sync(FULL, (overflow_arcs ? 2u : 0u) | (dirty ? 4u : 0u) | (vo.y ? 8u : 0u));
#endif
      // the chunk's real arcs staged slot-major (every lane's slot-0 arc, then slot 1, ...: one
      // ballot per inline slot) and relaxed 32 at a time (lane = arc); a chunk with more arcs than
      // the stage holds goes in two halves (lanes 0-15, then 16-31: <= 64 arcs each)
      const unsigned a0 = __ballot_sync(FULL, r0), a1 = __ballot_sync(FULL, r1);
      const unsigned a2 = __ballot_sync(FULL, r2), a3 = __ballot_sync(FULL, r3);
      const uint32_t n_all = __popc(a0) + __popc(a1) + __popc(a2) + __popc(a3);
#if GG_HALF_SPLIT
      const unsigned half = n_all > STAGE ? 0x0000FFFFu : FULL;
#else
      if (n_all > STAGE) OVF_RES(1);  // (rare: the chained level resumes it with its own stage)
      const unsigned half = FULL;
#endif
      for (unsigned pm = half;; pm = ~half) {
        const unsigned b0 = a0 & pm, b1 = a1 & pm, b2 = a2 & pm, b3 = a3 & pm;
        const uint32_t o1 = __popc(b0), o2 = o1 + __popc(b1), o3 = o2 + __popc(b2);
        const uint32_t n_arc = o3 + __popc(b3);
        if ((pm >> lane) & 1u) {
          if (r0) m.stage[__popc(b0 & lt)] = make_uint2(a01.x, du + a01.y);
          if (r1) m.stage[o1 + __popc(b1 & lt)] = make_uint2(a01.z, du + a01.w);
          if (r2) m.stage[o2 + __popc(b2 & lt)] = make_uint2(a23.x, du + a23.y);
          if (r3) m.stage[o3 + __popc(b3 & lt)] = make_uint2(a23.z, du + a23.w);
        }
        if (lane == 0) c_arcs += n_arc;
        __syncwarp();
        for (uint32_t j0 = 0; j0 < n_arc; j0 += 32) {
          bool has = false, ovf = false;
          uint32_t nslot = 0;
          if (j0 + lane < n_arc) {
            const uint2 a = m.stage[j0 + lane];
            bool imp;
            const int rr = tab_relax(m, H, a.x, a.y, imp);
            if (rr < 0) {
              ovf = true;
            } else if (imp) {
              mn = min(mn, a.y);
              const uint32_t bit = 1u << (rr & 31);
              if (!(atomicOr(&m.fin[rr >> 5], bit) & bit)) {
                has = true;
                nslot = (uint32_t)rr;
                prefetch_vertex(g, s, a.x);
              }
            }
          }
          if (__any_sync(FULL, ovf)) OVF_RES(2);
          const unsigned hm = __ballot_sync(FULL, has);
          if (nn + __popc(hm) > cp.F) OVF_RES(3);
          if (has) nfront[nn + __popc(hm & lt)] = nslot;
          nn += __popc(hm);
        }
        __syncwarp();  // (the stage is rewritten by the next half / chunk)
        if (pm != 0x0000FFFFu) break;  // (one part, or the second half done)
      }
#if GG_LATE_EVENTS
      // the chunk's harvest state (cell head, cleaned list, object index) is first used only now:
      // its loads' latency overlaps the relax passes above
      const bool dirty = harv && hd != NONE;
      const uint2 vo = harv ? vobj_valid(v0, cc) : make_uint2(0, 0);
      const uint32_t ev = __reduce_or_sync(FULL, (overflow_arcs ? 2u : 0u) | (dirty ? 4u : 0u) | (vo.y ? 8u : 0u));
#endif
      // vertices with more than 4 arcs: arcs 3.. from the CSR, one per lane per step (rare)
      if (ev & 2u) {
        uint32_t b0 = 0, b1 = 0;
        if (overflow_arcs) {
          b0 = g.rowptr[u] + 3;
          b1 = g.rowptr[u + 1];
        }
        const uint32_t most = __reduce_max_sync(FULL, b1 - b0);
        for (uint32_t j = 0; j < most; ++j) {
          bool has = false, ovf = false;
          uint32_t nslot = 0;
          if (b0 + j < b1) {
            const uint2 av = g.adj[b0 + j];
            ++c_arcs;
            const unsigned long long nd = (unsigned long long)du + av.y;
            if (nd < INF) {
              bool imp;
              const int rr = tab_relax(m, H, av.x, (uint32_t)nd, imp);
              if (rr < 0) {
                ovf = true;
              } else if (imp) {
                mn = min(mn, (uint32_t)nd);
                const uint32_t bit = 1u << (rr & 31);
                if (!(atomicOr(&m.fin[rr >> 5], bit) & bit)) {
                  has = true;
                  nslot = (uint32_t)rr;
                }
              }
            }
          }
          if (__any_sync(FULL, ovf)) OVF_RES(2);
          const unsigned hm = __ballot_sync(FULL, has);
          if (nn + __popc(hm) > cp.F) OVF_RES(3);
          if (has) nfront[nn + __popc(hm & lt)] = nslot;
          nn += __popc(hm);
        }
      }
      if (ev & 4u) {  // a cell with cached updates: lazy flush, then retry (Alg. 4 l.2-4)
        if (dirty) request_flush(s, hcell, P.epoch);
        request_lookahead(P, m, front, nf, lane);
        return RETRY;
      }
      c_harv += harv;
      if (track) {
        const uint32_t o = harv ? owner_of(hcell, g.n_cells, s.n_ranks) : s.rank;
        const unsigned long long bm = o != s.rank ? 1ull << o : 0ull;
        rmask |= ((unsigned long long)__reduce_or_sync(FULL, (uint32_t)(bm >> 32)) << 32) |
                 __reduce_or_sync(FULL, (uint32_t)bm);
      }
      if (ev & 8u) {  // harvest the objects of the vertices expanded for the first time
        const uint32_t most = __reduce_max_sync(FULL, vo.y);
        c_objs += vo.y;
        for (uint32_t j = 0; j < most; ++j) {
          bool hc = false;
          uint32_t ob = 0, oo = 0;
          if (j < vo.y) {
            const uint32_t p = vo.x + j;
            ob = s.ar.obj[p];
            const unsigned long long kk = s.ar.key[p];
            const uint32_t oe = s.ar.edge[p];
            oo = s.ar.off[p];
            const bool same_ahead = q.y > 0 && oe == q.x && oo >= q.y;  // already a candidate
            hc = !same_ahead && (!GG_HARVEST_VALIDATE || kk == s.ot_key[ob]);
          }
          if (!cand_push(m, nc, cp.C, hc, vslot, oo, ob, lt)) OVF_AT(4);
        }
      }
    }
#else
    // ---- 3. expand: 8 vertices per window, lane = (vertex, arc slot); the next window's
    //         global loads (inline arcs, object metadata) are issued before this window's
    //         relaxations
    auto load_win = [&](uint32_t w0) {
      Win w;
      const uint32_t vi = w0 + (lane >> 2), s4 = lane & 3;
      w.vv = vi < na;
      w.vslot = 0;
      w.u = 0;
      w.arc = make_uint2(0, 0);
      w.harv = false;
      w.hcell = 0;
      w.hd = NONE;
      w.cc = make_uint2(0, 0);
      w.v0 = make_uint2(0, 0);
      if (w.vv) {
        w.vslot = m.act[vi];
        w.u = KEYR(m, w.vslot);
        w.arc = g.vadj[(size_t)w.u * 4 + s4];
        if (s4 == 0) {
          w.hcell = cellof(g, w.u);
          w.hd = s.cell_head[w.hcell];
          w.cc = s.cell_comp[w.hcell];
          if (!GG_VHAS || vhas_bit(s, w.u)) w.v0 = s.v_obj[w.u];
          w.harv = !(atomicOr(&m.listed[w.vslot >> 5], 1u << (w.vslot & 31)) & (1u << (w.vslot & 31)));
        }
      }
      return w;
    };
    Win cur = load_win(0);
    for (uint32_t w0 = 0; w0 < na; w0 += 8) {
      const Win nxt = load_win(w0 + 8);  // (all lanes out of range past the last window)
      // D re-read now: an earlier window may have improved it (the frontier bit was cleared
      // at partition, so such an improvement also re-queued the vertex)
      const uint32_t du = cur.vv ? DISTR(m, cur.vslot) : INF;
      bool has = false, ovf = false;
      uint32_t nslot = 0;
      auto relax = [&](uint32_t dst, uint32_t w) {
        ++c_arcs;
        const unsigned long long nd = (unsigned long long)du + w;
        if (nd >= INF) return;
        bool imp;
        const int rr = tab_relax(m, H, dst, (uint32_t)nd, imp);
        if (rr < 0) {
          ovf = true;
        } else if (imp) {
          mn = min(mn, (uint32_t)nd);
          const uint32_t bit = 1u << (rr & 31);
          if (!(atomicOr(&m.fin[rr >> 5], bit) & bit)) {
            has = true;
            nslot = (uint32_t)rr;
            prefetch_vertex(g, s, dst);
          }
        }
      };
      const bool overflow_arcs = cur.arc.y == WMAX;
      if (cur.arc.y != 0 && !overflow_arcs) relax(cur.arc.x, cur.arc.y);
      // harvest the objects of the vertices expanded for the first time; a cell with cached
      // updates must be cleaned first (lazy flush): request it and retry the query
      const bool dirty = cur.harv && cur.hd != NONE;
      const uint2 vo = cur.harv ? vobj_valid(cur.v0, cur.cc) : make_uint2(0, 0);
      // one warp vote for every rare event of the window
      const uint32_t ev = __reduce_or_sync(FULL, (ovf ? 1u : 0u) | (overflow_arcs ? 2u : 0u) |
                                                     (dirty ? 4u : 0u) | (vo.y ? 8u : 0u));
      if (ev & 1u) return OVERFLOW;
      unsigned hm = __ballot_sync(FULL, has);
      if (nn + __popc(hm) > cp.F) return OVERFLOW;
      if (has) nfront[nn + __popc(hm & lt)] = nslot;
      nn += __popc(hm);
      // vertices with more than 4 arcs: the rest live in the CSR (rare on road graphs)
      if (ev & 2u) {
        uint32_t a0 = 0, a1 = 0;
        if (overflow_arcs) {
          a0 = g.rowptr[cur.u] + 3;
          a1 = g.rowptr[cur.u + 1];
        }
        const uint32_t most = __reduce_max_sync(FULL, a1 - a0);
        for (uint32_t j = 0; j < most; ++j) {
          has = false;
          ovf = false;
          if (a0 + j < a1) {
            const uint2 av = g.adj[a0 + j];
            relax(av.x, av.y);
          }
          if (__any_sync(FULL, ovf)) return OVERFLOW;
          hm = __ballot_sync(FULL, has);
          if (nn + __popc(hm) > cp.F) return OVERFLOW;
          if (has) nfront[nn + __popc(hm & lt)] = nslot;
          nn += __popc(hm);
        }
      }
      if (ev & 4u) {
        if (dirty) request_flush(s, cur.hcell, P.epoch);
        request_lookahead(P, m, front, nf, lane);
        return RETRY;
      }
      c_harv += cur.harv;
      if (track) {
        const uint32_t o = cur.harv ? owner_of(cur.hcell, g.n_cells, s.n_ranks) : s.rank;
        const unsigned long long bm = o != s.rank ? 1ull << o : 0ull;
        rmask |= ((unsigned long long)__reduce_or_sync(FULL, (uint32_t)(bm >> 32)) << 32) |
                 __reduce_or_sync(FULL, (uint32_t)bm);
      }
      if (ev & 8u) {
        const uint32_t most = __reduce_max_sync(FULL, vo.y);
        c_objs += vo.y;
        for (uint32_t j = 0; j < most; ++j) {
          bool hc = false;
          uint32_t ob = 0, oo = 0;
          if (j < vo.y) {
            const uint32_t p = vo.x + j;
            ob = s.ar.obj[p];
            const unsigned long long kk = s.ar.key[p];
            const uint32_t oe = s.ar.edge[p];
            oo = s.ar.off[p];
            const bool same_ahead = q.y > 0 && oe == q.x && oo >= q.y;  // already a candidate
            hc = !same_ahead && (!GG_HARVEST_VALIDATE || kk == s.ot_key[ob]);
          }
          if (!cand_push(m, nc, cp.C, hc, cur.vslot, oo, ob, lt)) return OVERFLOW;
        }
      }
      cur = nxt;
    }
#endif
    auto* tmp = front;
    front = nfront;
    nfront = tmp;
    nf = nn;
    blo = __reduce_min_sync(FULL, mn);
    __syncwarp();
  }
  c_arcs = __reduce_add_sync(FULL, c_arcs);
  c_harv = __reduce_add_sync(FULL, c_harv);
  c_objs = __reduce_add_sync(FULL, c_objs);

  // ---- 4. the k smallest (dist, obj) ------------------------------------------------------
  if (GG_REG_SORT && nc <= 32 && k <= 32) {  // one candidate per lane: bitonic sort by shuffles
    unsigned long long v = EMPTY64;
    if (lane < nc) {
      const unsigned long long d = cand_dist(m, lane);
      if (d < INF) v = (d << 32) | m.cobj[lane];
    }
#pragma unroll
    for (uint32_t size = 2; size <= 32; size <<= 1) {
#pragma unroll
      for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
        const unsigned long long o = __shfl_xor_sync(FULL, v, stride);
        const bool keep_min = ((lane & stride) == 0) == ((lane & size) == 0);
        v = keep_min ? min(v, o) : max(v, o);
      }
    }
    if (lane < k) {
      const bool ok = v != EMPTY64 && (uint32_t)(v >> 32) <= lim;
      P.out_obj[(size_t)qi * k + lane] = ok ? (uint32_t)v : GGRID_PAD;
      P.out_dist[(size_t)qi * k + lane] = ok ? (uint32_t)(v >> 32) : GGRID_PAD;
    }
    goto finish;
  }
  for (uint32_t i = lane; i < nc; i += 32) {
    const unsigned long long d = cand_dist(m, i);
    m.cand[i] = d < INF ? ((d << 32) | m.cobj[i]) : EMPTY64;
  }
  __syncwarp();
  warp_sort(m.cand, nc, cp.C, lane);
  for (uint32_t r = lane; r < k; r += 32) {
    const unsigned long long dk = r < nc ? m.cand[r] : EMPTY64;
    const bool ok = dk != EMPTY64 && (uint32_t)(dk >> 32) <= lim;
    P.out_obj[(size_t)qi * k + r] = ok ? (uint32_t)dk : GGRID_PAD;
    P.out_dist[(size_t)qi * k + r] = ok ? (uint32_t)(dk >> 32) : GGRID_PAD;
  }
finish:
  if (lane == 0 && P.remote) P.remote[qi] = rmask;
  if (lane == 0) {
    atomicAdd(&s.st->ex_iters, (unsigned long long)c_iter);
    atomicAdd(&s.st->ex_vertices, (unsigned long long)c_vert);
    atomicAdd(&s.st->ex_arcs, (unsigned long long)c_arcs);
    atomicAdd(&s.st->ex_harvested, (unsigned long long)c_harv);
    atomicAdd(&s.st->ex_objects, (unsigned long long)c_objs);
  }
  return DONE;
}

// SMEM: the working memory is this CTA's shared memory (levels 0..L-2), else per-warp global
// scratch (the last level).  Two instantiations, so that every table access of the shared one
// compiles to LDS/STS/ATOMS with 32-bit addresses (one pointer that may be either space makes
// them generic 64-bit LD/ST/ATOM, measured ~10% slower overall).
// registers capped for GG_WARP_MINB resident CTAs of 4 queries per SM: the 600-slot table makes a
// query 7,008 B of shared memory, so 8 CTAs (32 queries) fit and 64 registers must too
#ifndef GG_WARP_MINB
#define GG_WARP_MINB 8
#endif
#define GG_EXPAND_BOUNDS __launch_bounds__(128, GG_WARP_MINB)
template <bool SMEM>
__global__ void GG_EXPAND_BOUNDS k_expand(QParams P) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int lane = threadIdx.x & 31;
  const uint32_t warp = threadIdx.x >> 5;
  using S = typename std::conditional<SMEM, uint16_t, uint32_t>::type;
  const size_t wbytes = (warpmem_bytes(P.caps, sizeof(S)) + 15) & ~size_t(15);
  const uint32_t gw = blockIdx.x * P.warps_per_cta + warp;
  unsigned char* base = SMEM ? smem_raw + (size_t)warp * wbytes : P.scratch + (size_t)gw * wbytes;
  const WarpMemT<S> m = carve<S>(base, P.caps);
  pdl_trigger(P);
  for (;;) {  // persistent: queries fetched dynamically
    uint32_t li = 0;
    if (lane == 0) li = atomicAdd(&P.s.st->expand_work[P.level], 1u);
    li = __shfl_sync(0xffffffffu, li, 0);
    if (li >= P.n) break;
    const uint32_t qi = P.qlist ? P.qlist[li] : li;
    Resume rs;
    rs.ok = false;
    rs.rmask = 0;
    const int r = run_query(P, m, qi, lane, rs);
    if (SMEM && r == OVERFLOW && P.resume) {
      promote_export(P, m, qi, lane, rs);
    } else if (lane == 0 && r != DONE) {
      finish_undone(P, qi, r);
    }
    __syncwarp();
  }
  __syncthreads();  // (the chained level waits for every CTA -- all of its warps -- to exit)
  if (threadIdx.x == 0) count_exit(P);
}

// ---------------------------------------------------------------------------------------------
// Paired variant of the one-warp kernel (GG_PAIR): each half-warp (16 lanes) runs its own query
// with its own shared-memory table, and the two halves execute every phase of a round -- the
// termination test, the frontier partition, the chunk load + arc compaction, the relax passes and
// the harvest -- in the same instructions, each on its own data (loop bounds are the larger of
// the two halves'; half-warp ballots, shuffles and reductions).  A round's bucket (~14 vertices at
// C3) and its arcs (~34) fill 16-lane passes far better than 32-lane ones, so a query costs fewer
// warp instructions; the queries resident per SM are the same (shared memory per query).  A half
// whose query ends fetches the next one while the other continues.  Same arithmetic and outcome
// rules as run_query (DONE / RETRY / OVERFLOW).
#ifndef GG_PAIR
#define GG_PAIR 0
#endif

struct HalfWarp {
  uint32_t h, hl, base;
  unsigned mask, lt;
};
__device__ __forceinline__ uint32_t hsum(const HalfWarp& W, uint32_t x) {
#pragma unroll
  for (int o = 8; o > 0; o >>= 1) x += __shfl_xor_sync(W.mask, x, o);
  return x;
}
__device__ __forceinline__ uint32_t hmin(const HalfWarp& W, uint32_t x) {
#pragma unroll
  for (int o = 8; o > 0; o >>= 1) x = min(x, __shfl_xor_sync(W.mask, x, o));
  return x;
}
__device__ __forceinline__ uint32_t hmax(const HalfWarp& W, uint32_t x) {
#pragma unroll
  for (int o = 8; o > 0; o >>= 1) x = max(x, __shfl_xor_sync(W.mask, x, o));
  return x;
}
__device__ __forceinline__ uint32_t hor(const HalfWarp& W, uint32_t x) {
#pragma unroll
  for (int o = 8; o > 0; o >>= 1) x |= __shfl_xor_sync(W.mask, x, o);
  return x;
}
// full-warp forms for the phases both halves run in the same instructions
__device__ __forceinline__ uint32_t horF(const HalfWarp&, uint32_t x) {
#pragma unroll
  for (int o = 8; o > 0; o >>= 1) x |= __shfl_xor_sync(0xffffffffu, x, o);
  return x;
}
__device__ __forceinline__ uint32_t hmaxF(const HalfWarp&, uint32_t x) {
#pragma unroll
  for (int o = 8; o > 0; o >>= 1) x = max(x, __shfl_xor_sync(0xffffffffu, x, o));
  return x;
}
// the larger of the two halves' (half-uniform) values: the shared loop bound of a phase
__device__ __forceinline__ uint32_t both_max(uint32_t v) { return max(v, __shfl_xor_sync(0xffffffffu, v, 16)); }

__device__ __forceinline__ bool cand_push16(const WarpMemS& m, const HalfWarp& W, uint32_t& nc, uint32_t C, bool has,
                                            uint32_t slot, uint32_t off, uint32_t obj) {
  const unsigned hm = __ballot_sync(W.mask, has) & W.mask;
  if (!hm) return true;
  if (nc + __popc(hm) > C) return false;
  if (has) {
    const uint32_t i = nc + __popc(hm & W.lt);
    m.cand[i] = ((unsigned long long)slot << 32) | off;
    m.cobj[i] = obj;
  }
  nc += __popc(hm);
  return true;
}

__device__ __forceinline__ bool cand_push16F(const WarpMemS& m, const HalfWarp& W, uint32_t& nc, uint32_t C, bool has,
                                             uint32_t slot, uint32_t off, uint32_t obj) {
  const unsigned hm = __ballot_sync(0xffffffffu, has) & W.mask;
  if (hm && nc + __popc(hm) > C) return false;
  if (has) {
    const uint32_t i = nc + __popc(hm & W.lt);
    m.cand[i] = ((unsigned long long)slot << 32) | off;
    m.cobj[i] = obj;
  }
  nc += __popc(hm);
  return true;
}

__device__ void half_sort(unsigned long long* a, uint32_t n, uint32_t cap, const HalfWarp& W) {
  uint32_t n2 = 1;
  while (n2 < n) n2 <<= 1;
  if (n2 > cap) n2 = cap;
  for (uint32_t i = n + W.hl; i < n2; i += 16) a[i] = EMPTY64;
  __syncwarp(W.mask);
  for (uint32_t size = 2; size <= n2; size <<= 1) {
    for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
      for (uint32_t i = W.hl; i < n2 / 2; i += 16) {
        const uint32_t lo = 2 * i - (i & (stride - 1));
        const uint32_t hi = lo + stride;
        const bool asc = (lo & size) == 0;
        const unsigned long long x = a[lo], y = a[hi];
        if ((x > y) == asc) {
          a[lo] = y;
          a[hi] = x;
        }
      }
      __syncwarp(W.mask);
    }
  }
}

__global__ void k_expand_pair(QParams P) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const DevGraph& g = P.g;
  const DevState& s = P.s;
  const Caps cp = P.caps;
  const uint32_t H = cp.H, k = P.k;
  const int lane = threadIdx.x & 31;
  const uint32_t warp = threadIdx.x >> 5;
  HalfWarp W;
  W.h = (uint32_t)lane >> 4;
  W.hl = (uint32_t)lane & 15u;
  W.base = W.h * 16;
  W.mask = 0xFFFFu << W.base;
  W.lt = lanemask_lt() & W.mask;
  const size_t wbytes = (warpmem_bytes(cp, 2) + 15) & ~size_t(15);
  const WarpMemS m = carve<uint16_t>(smem_raw + (size_t)(2 * warp + W.h) * wbytes, cp);
  pdl_trigger(P);
  const bool track = P.remote != nullptr && s.n_ranks > 1;

  // per-half (half-uniform) query state
  uint32_t qi = NONE;
  bool need = true, exhausted = false;
  uint2 q = make_uint2(0, 0), ei = make_uint2(0, 0);
  uint32_t lim = INF, nf = 0, nc = 0, blo = 0, fb = 0;
  unsigned long long rmask = 0;
  uint32_t c_iter = 0, c_vert = 0, c_arcs = 0, c_harv = 0, c_objs = 0;
  int outcome = -1;  // set when the query ends (DONE / RETRY / OVERFLOW)

  auto finish = [&](int r) {  // (half-divergent) write the answer or queue the query; fetch next
    if (r == DONE && qi != NONE) {
      for (uint32_t i = W.hl; i < nc; i += 16) {
        const unsigned long long d = cand_dist(m, i);
        m.cand[i] = d < INF ? ((d << 32) | m.cobj[i]) : EMPTY64;
      }
      __syncwarp(W.mask);
      half_sort(m.cand, nc, cp.C, W);
      for (uint32_t r2 = W.hl; r2 < k; r2 += 16) {
        const unsigned long long dk = r2 < nc ? m.cand[r2] : EMPTY64;
        const bool ok = dk != EMPTY64 && (uint32_t)(dk >> 32) <= lim;
        P.out_obj[(size_t)qi * k + r2] = ok ? (uint32_t)dk : GGRID_PAD;
        P.out_dist[(size_t)qi * k + r2] = ok ? (uint32_t)(dk >> 32) : GGRID_PAD;
      }
      const unsigned long long rm = ((unsigned long long)hor(W, (uint32_t)(rmask >> 32)) << 32) | hor(W, (uint32_t)rmask);
      const uint32_t sa = hsum(W, c_arcs), sh = hsum(W, c_harv), so = hsum(W, c_objs);
      if (W.hl == 0) {
        if (P.remote) P.remote[qi] = rm;
        atomicAdd(&s.st->ex_iters, (unsigned long long)c_iter);
        atomicAdd(&s.st->ex_vertices, (unsigned long long)c_vert);
        atomicAdd(&s.st->ex_arcs, (unsigned long long)sa);
        atomicAdd(&s.st->ex_harvested, (unsigned long long)sh);
        atomicAdd(&s.st->ex_objects, (unsigned long long)so);
      }
    } else if (qi != NONE && W.hl == 0) {
      finish_undone(P, qi, r);
    }
    __syncwarp(W.mask);
    need = true;
  };

  for (;;) {
    // ---- A. a half without a query fetches and starts the next one
    while (need && !exhausted) {
      uint32_t li = 0;
      if (W.hl == 0) li = atomicAdd(&s.st->expand_work[P.level], 1u);
      li = __shfl_sync(W.mask, li, W.base);
      if (li >= P.n) {
        exhausted = true;
        qi = NONE;
        break;
      }
      qi = P.qlist ? P.qlist[li] : li;
      need = false;
      outcome = -1;
      for (uint32_t i = W.hl; i < H; i += 16) {
        KEYR(m, i) = EMPTY32;
        DISTR(m, i) = INF;
      }
      for (uint32_t i = W.hl; i < (H + 31) / 32; i += 16) {
        m.fin[i] = 0;
        m.listed[i] = 0;
      }
      __syncwarp(W.mask);
      c_iter = c_vert = c_arcs = c_harv = c_objs = 0;
      nc = 0;
      rmask = 0;
      fb = 0;
      q = P.q[qi];
      if (q.x >= g.A) {  // invalid query: reported by the seed kernel (EINVAL)
        need = true;
        continue;
      }
      ei = g.einfo[q.x];
      if (q.y >= ei.y) {
        need = true;
        continue;
      }
      lim = P.bound ? P.bound[qi] : INF;
      if (track) {
        const uint32_t o = owner_of(cellof(g, ei.x), g.n_cells, s.n_ranks);
        if (o != s.rank) rmask |= 1ull << o;
      }
      const uint32_t seed_v = q.y == 0 ? ei.x : g.edst[q.x];
      const uint32_t seed_d = q.y == 0 ? 0u : ei.y - q.y;
      if (W.hl == 0) {
        bool imp;
        const int sl = tab_relax(m, H, seed_v, seed_d, imp);
        m.front0[0] = (uint32_t)sl;
        m.fin[sl >> 5] |= 1u << (sl & 31);
      }
      __syncwarp(W.mask);
      nf = 1;
      blo = seed_d;
      if (q.y > 0) {  // objects on q's own arc ahead of q (reading R2), stored at src(q.e)
        const uint32_t c = cellof(g, ei.x);
        if (s.cell_head[c] != NONE) {
          if (W.hl == 0) request_flush(s, c, P.epoch);
          finish(RETRY);
          continue;
        }
        const uint2 vo = vobj_valid(s.v_obj[ei.x], s.cell_comp[c]);
        bool ovf = false;
        for (uint32_t j0 = 0; j0 < vo.y && !ovf; j0 += 16) {
          const uint32_t j = j0 + W.hl;
          bool has = false;
          uint32_t ob = 0, dd = 0;
          if (j < vo.y) {
            const uint32_t pp = vo.x + j;
            ob = s.ar.obj[pp];
            const uint32_t oe = s.ar.edge[pp], oo = s.ar.off[pp];
            if (oe == q.x && oo >= q.y && valid_rec(s, pp, ob)) {
              has = true;
              dd = oo - q.y;
            }
          }
          ovf = !cand_push16(m, W, nc, cp.C, has, SPECIAL, dd, ob);
        }
        if (ovf) {
          finish(OVERFLOW);
          continue;
        }
      }
    }
    if (__all_sync(0xffffffffu, exhausted)) break;
    bool act = !exhausted;

    // ---- B. termination: k candidates strictly closer than anything not yet final (both
    //         halves count in the same instructions; only the finish is per half)
    {
      if (act) ++c_iter;
      const bool early = act && (nf == 0 || blo > lim);
      const bool chk = act && !early && nc >= k;
      const uint32_t nc_b = both_max(chk ? nc : 0u);
      uint32_t cl = 0;
      for (uint32_t i = W.hl; i < nc_b; i += 16)
        if (chk && i < nc) cl += cand_dist(m, i) < blo;
#pragma unroll
      for (int o = 8; o > 0; o >>= 1) cl += __shfl_xor_sync(0xffffffffu, cl, o);
      if (early || (chk && cl >= k)) {
        finish(DONE);
        act = false;
      }
    }
    auto* front = fb ? m.front1 : m.front0;
    auto* nfront = fb ? m.front0 : m.front1;

    // ---- C. partition: the bucket [blo, blo + delta) into act, the rest re-queued
    const uint32_t bhi = (blo > INF - g.delta) ? INF : blo + g.delta;
    uint32_t nn = 0, na = 0, mn = INF;
    const uint32_t nf_b = both_max(act ? nf : 0u);
    for (uint32_t b0 = 0; b0 < nf_b; b0 += 16) {
      const uint32_t i = b0 + W.hl;
      const uint32_t sl = (act && i < nf) ? front[i] : NONE;
      const uint32_t ent = sl != NONE ? DISTR(m, sl) : INF;
      const bool a = sl != NONE && ent < bhi;
      const bool r = sl != NONE && !a;
      const unsigned rm = __ballot_sync(0xffffffffu, r) & W.mask;
      if (r) {
        nfront[nn + __popc(rm & W.lt)] = sl;
        mn = min(mn, ent);
      }
      nn += __popc(rm);
      const unsigned am = __ballot_sync(0xffffffffu, a) & W.mask;
      if (a) {
        m.act[na + __popc(am & W.lt)] = sl;
        atomicAnd(&m.fin[sl >> 5], ~(1u << (sl & 31)));
      }
      na += __popc(am);
    }
    __syncwarp();
    if (act) c_vert += na;

    // ---- D. expand the bucket in chunks of 16 vertices, lane = vertex; arcs compacted
    int oc = -1;  // this half's outcome met in the round (RETRY / OVERFLOW)
    const uint32_t na_b = both_max(na);
    for (uint32_t c0 = 0; c0 < na_b; c0 += 16) {
      const uint32_t vi = c0 + W.hl;
      const bool vv = oc < 0 && vi < na;
      uint32_t vslot = 0, u = 0, du = INF, hcell = 0, hd = NONE;
      uint4 a01 = make_uint4(0, 0, 0, 0), a23 = make_uint4(0, 0, 0, 0);
      uint2 cc = make_uint2(0, 0), v0 = make_uint2(0, 0);
      bool harv = false;
      if (vv) {
        vslot = m.act[vi];
        u = KEYR(m, vslot);
        du = DISTR(m, vslot);
        const uint4* rec = reinterpret_cast<const uint4*>(g.vadj + (size_t)u * 4);
        a01 = rec[0];
        a23 = rec[1];
        harv = !(atomicOr(&m.listed[vslot >> 5], 1u << (vslot & 31)) & (1u << (vslot & 31)));
        if (harv) {
          hcell = cellof(g, u);
          hd = s.cell_head[hcell];
          cc = s.cell_comp[hcell];
          if (!GG_VHAS || vhas_bit(s, u)) v0 = s.v_obj[u];
        }
      }
      const bool overflow_arcs = a23.w == WMAX;
      const uint32_t room = INF - du;
      auto real = [&](uint32_t w) { return (w - 1u < WMAX - 1u) & (w < room); };
      const uint32_t r0 = real(a01.y), r1 = real(a01.w), r2 = real(a23.y), r3 = real(a23.w);
      const uint32_t cnt = r0 + r1 + r2 + r3;
      uint32_t pre = cnt;
#pragma unroll
      for (int o = 1; o < 16; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, pre, o, 16);
        if (W.hl >= (uint32_t)o) pre += y;
      }
      const uint32_t n_arc = __shfl_sync(0xffffffffu, pre, W.base + 15);
      pre -= cnt;
      if (r0) m.stage[pre++] = make_uint2(a01.x, du + a01.y);
      if (r1) m.stage[pre++] = make_uint2(a01.z, du + a01.w);
      if (r2) m.stage[pre++] = make_uint2(a23.x, du + a23.y);
      if (r3) m.stage[pre++] = make_uint2(a23.z, du + a23.w);
      c_arcs += cnt;
      const bool dirty = harv && hd != NONE;
      const uint2 vo = harv ? vobj_valid(v0, cc) : make_uint2(0, 0);
      const uint32_t ev = horF(W, (overflow_arcs ? 2u : 0u) | (dirty ? 4u : 0u) | (vo.y ? 8u : 0u));
      __syncwarp();
      // relax: lane = arc of this half's staged list
      const uint32_t narc_b = both_max(n_arc);
      for (uint32_t j0 = 0; j0 < narc_b; j0 += 16) {
        bool has = false, ovf = false;
        uint32_t nslot = 0;
        if (j0 + W.hl < n_arc) {
          const uint2 a = m.stage[j0 + W.hl];
          bool imp;
          const int rr = tab_relax(m, H, a.x, a.y, imp);
          if (rr < 0) {
            ovf = true;
          } else if (imp) {
            mn = min(mn, a.y);
            const uint32_t bit = 1u << (rr & 31);
            if (!(atomicOr(&m.fin[rr >> 5], bit) & bit)) {
              has = true;
              nslot = (uint32_t)rr;
              prefetch_vertex(g, s, a.x);
            }
          }
        }
        const unsigned ob_ = __ballot_sync(0xffffffffu, ovf) & W.mask;
        const unsigned hm = __ballot_sync(0xffffffffu, has) & W.mask;
        if (oc < 0 && (ob_ || nn + __popc(hm) > cp.F)) oc = OVERFLOW;
        if (oc < 0) {
          if (has) nfront[nn + __popc(hm & W.lt)] = nslot;
          nn += __popc(hm);
        }
      }
      __syncwarp();  // (the stage / source map is rewritten by the next chunk)
      // vertices with more than 4 arcs: arcs 3.. from the CSR, one per lane per step (rare)
      if (both_max(ev & 2u)) {
        uint32_t b0 = 0, b1 = 0;
        if (overflow_arcs && oc < 0) {
          b0 = g.rowptr[u] + 3;
          b1 = g.rowptr[u + 1];
        }
        const uint32_t most = both_max(hmaxF(W, b1 - b0));
        for (uint32_t j = 0; j < most; ++j) {
          bool has = false, ovf = false;
          uint32_t nslot = 0;
          if (b0 + j < b1) {
            const uint2 av = g.adj[b0 + j];
            ++c_arcs;
            const unsigned long long nd = (unsigned long long)du + av.y;
            if (nd < INF) {
              bool imp;
              const int rr = tab_relax(m, H, av.x, (uint32_t)nd, imp);
              if (rr < 0) {
                ovf = true;
              } else if (imp) {
                mn = min(mn, (uint32_t)nd);
                const uint32_t bit = 1u << (rr & 31);
                if (!(atomicOr(&m.fin[rr >> 5], bit) & bit)) {
                  has = true;
                  nslot = (uint32_t)rr;
                }
              }
            }
          }
          const unsigned ob_ = __ballot_sync(0xffffffffu, ovf) & W.mask;
          const unsigned hm = __ballot_sync(0xffffffffu, has) & W.mask;
          if (oc < 0 && (ob_ || nn + __popc(hm) > cp.F)) oc = OVERFLOW;
          if (oc < 0) {
            if (has) nfront[nn + __popc(hm & W.lt)] = nslot;
            nn += __popc(hm);
          }
        }
      }
      if (oc < 0 && (ev & 4u)) {  // a cell with cached updates: lazy flush, then retry
        if (dirty) request_flush(s, hcell, P.epoch);
        for (uint32_t i = W.hl; i < nf; i += 16) request_flush(s, cellof(g, KEYR(m, front[i])), P.epoch);
        oc = RETRY;
      }
      if (oc < 0) {
        c_harv += harv;
        if (track) {
          const uint32_t o = harv ? owner_of(hcell, g.n_cells, s.n_ranks) : s.rank;
          if (o != s.rank) rmask |= 1ull << o;
        }
      }
      if (both_max(oc < 0 ? (ev & 8u) : 0u)) {  // harvest the objects of first-expanded vertices
        const uint32_t vmx = hmaxF(W, vo.y);  // (every lane of both halves runs the full-warp shuffles)
        const uint32_t most = both_max(oc < 0 ? vmx : 0u);
        if (oc < 0) c_objs += vo.y;
        for (uint32_t j = 0; j < most; ++j) {
          bool hc = false;
          uint32_t ob = 0, oo = 0;
          if (oc < 0 && j < vo.y) {
            const uint32_t pp = vo.x + j;
            ob = s.ar.obj[pp];
            const uint32_t oe = s.ar.edge[pp];
            oo = s.ar.off[pp];
            const bool same_ahead = q.y > 0 && oe == q.x && oo >= q.y;  // already a candidate
            hc = !same_ahead && valid_rec(s, pp, ob);
          }
          const bool okp = cand_push16F(m, W, nc, cp.C, hc, vslot, oo, ob);
          if (!okp && oc < 0) oc = OVERFLOW;
        }
      }
    }
    // ---- E. round end
    uint32_t mnh = mn;
#pragma unroll
    for (int o = 8; o > 0; o >>= 1) mnh = min(mnh, __shfl_xor_sync(0xffffffffu, mnh, o));
    if (oc >= 0) {
      finish(oc);
    } else if (act) {
      nf = nn;
      blo = mnh;
      fb ^= 1u;
    }
    __syncwarp();
  }
  __syncthreads();  // (the chained level waits for every CTA to exit)
  if (threadIdx.x == 0) count_exit(P);
}

// ---------------------------------------------------------------------------------------------
// CTA-per-query variant: the same expansion with W warps cooperating on one query (block-wide
// shared-memory table, atomically appended frontier and candidates, barriers between the
// phases of a round).  Used where one warp is too narrow: balls of thousands of vertices (the
// larger levels, whose per-query tables would otherwise leave one or a few warps per SM) and
// small batches, where the single query's latency is the metric ("G-Grid (L)", P@61891).
template <int W>
struct CtaShared {
  uint32_t nn[2], na[2];  // next-frontier and bucket sizes, by round parity (a round's counters
                          // are reset one round later, when every thread has read them)
  uint32_t stop[2];       // termination verdict (k candidates closer than the frontier), by parity
  uint32_t nc;            // candidates
  uint32_t flags;         // FL_RETRY (a dirty cell met) | FL_OVF (a capacity exceeded)
  uint32_t red[2][W];     // per-warp next-frontier minimum, by round parity
  uint32_t sum[W];
  unsigned long long redl[W];
};
constexpr uint32_t FL_RETRY = 1, FL_OVF = 2;

template <int W>
__device__ __forceinline__ uint32_t block_sum(uint32_t v, CtaShared<W>& sh) {
  v = __reduce_add_sync(0xffffffffu, v);
  __syncthreads();
  if ((threadIdx.x & 31) == 0) sh.sum[threadIdx.x >> 5] = v;
  __syncthreads();
  uint32_t r = 0;
#pragma unroll
  for (int w = 0; w < W; ++w) r += sh.sum[w];
  return r;
}

// block bitonic sort of a[0..n) ascending (n padded to a power of two <= cap)
template <int W>
__device__ void block_sort(unsigned long long* a, uint32_t n, uint32_t cap) {
  constexpr uint32_t T = W * 32;
  uint32_t n2 = 1;
  while (n2 < n) n2 <<= 1;
  if (n2 > cap) n2 = cap;
  for (uint32_t i = n + threadIdx.x; i < n2; i += T) a[i] = EMPTY64;
  __syncthreads();
  for (uint32_t size = 2; size <= n2; size <<= 1) {
    for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
      for (uint32_t i = threadIdx.x; i < n2 / 2; i += T) {
        const uint32_t lo = 2 * i - (i & (stride - 1));
        const uint32_t hi = lo + stride;
        const bool asc = (lo & size) == 0;
        const unsigned long long x = a[lo], y = a[hi];
        if ((x > y) == asc) {
          a[lo] = y;
          a[hi] = x;
        }
      }
      __syncthreads();
    }
  }
}

// Capacities of a level: compile-time (constant shared-memory offsets and bounds: no registers
// hold the working-memory pointers), or from the launch parameters.
struct DynCaps {
  __device__ static Caps get(const QParams& P) { return P.caps; }
};
template <uint32_t H_, uint32_t F_, uint32_t C_>
struct FixCaps {
  static_assert((C_ & (C_ - 1)) == 0, "candidate capacity must be a power of two");
  __host__ __device__ static constexpr Caps get(const QParams&) { return Caps{H_, F_, C_}; }
  static constexpr Caps caps() { return Caps{H_, F_, C_}; }
};

template <int W, class CP>
__device__ int run_query_cta(const QParams& P, const WarpMemS& m, CtaShared<W>& sh, uint32_t qi,
                             uint32_t rslot) {
  constexpr uint32_t T = W * 32;
  const unsigned FULL = 0xffffffffu;
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const DevGraph& g = P.g;
  const DevState& s = P.s;
  const Caps cp = CP::get(P);
  const uint32_t H = cp.H;
  const uint32_t k = P.k;

  for (uint32_t i = tid; i < H; i += T) {
    KEYR(m, i) = EMPTY32;
    DISTR(m, i) = INF;
  }
  for (uint32_t i = tid; i < (H + 31) / 32; i += T) m.fin[i] = 0;
  for (uint32_t i = tid; i < (H + 31) / 32; i += T) m.listed[i] = 0;
  if (tid == 0) {
    sh.nn[0] = sh.nn[1] = sh.na[0] = sh.na[1] = 0;
    sh.stop[0] = sh.stop[1] = 0;
    sh.nc = 0;
    sh.flags = 0;
  }
  __syncthreads();

  const uint2 q = P.q[qi];
  if (q.x >= g.A) return DONE;
  const uint2 ei = g.einfo[q.x];
  if (q.y >= ei.y) return DONE;
  const uint32_t lim = P.bound ? P.bound[qi] : INF;
  const bool track = P.remote != nullptr && s.n_ranks > 1;
  unsigned long long rmask = 0;  // (per thread; OR-reduced at the end)
  if (track) {
    const uint32_t o = owner_of(cellof(g, ei.x), g.n_cells, s.n_ranks);
    if (o != s.rank) rmask |= 1ull << o;
  }
  const uint32_t seed_d = q.y == 0 ? 0u : ei.y - q.y;
  uint32_t nf = 1, blo = seed_d;
  // a query promoted with its state (promote_export): the record's table, frontier (its fin
  // bits plus the unexpanded rest of its bucket), listed bits and candidates are re-hashed into
  // this level's table, and the search continues from there
  const RecView rv = rslot != NONE ? rec_view(P.resume + (size_t)rslot * P.resume_bytes, P.rcaps) : RecView{};
  const bool resumed = rslot != NONE && __ldcg(&rv.hdr->valid) == 1u && __ldcg(&rv.hdr->qi) == qi;
  if (resumed) {
    const uint32_t H0 = P.rcaps.H;
    for (uint32_t i = tid; i < H0; i += T) {
      const uint32_t v = __ldcg(rv.key + i);
      if (v == EMPTY32) continue;
      bool imp;
      const int sl = tab_relax(m, H, v, __ldcg(rv.dist + i), imp);
      if (sl < 0) {
        atomicOr(&sh.flags, FL_OVF);
        continue;
      }
      const uint32_t bit = 1u << (sl & 31);
      if (__ldcg(rv.listed + (i >> 5)) & (1u << (i & 31))) atomicOr(&m.listed[sl >> 5], bit);
      if ((__ldcg(rv.fin + (i >> 5)) & (1u << (i & 31))) && !(atomicOr(&m.fin[sl >> 5], bit) & bit)) {
        const uint32_t p = atomicAdd(&sh.nn[1], 1u);
        if (p < cp.F) m.front0[p] = (uint16_t)sl;
      }
    }
    __syncthreads();
    const uint32_t n_act = __ldcg(&rv.hdr->n_act), nc0 = __ldcg(&rv.hdr->nc);
    for (uint32_t j = tid; j < n_act; j += T) {
      const int sl = tab_find(m, H, __ldcg(rv.key + __ldcg(rv.act + j)));
      if (sl < 0) {
        atomicOr(&sh.flags, FL_OVF);
        continue;
      }
      const uint32_t bit = 1u << (sl & 31);
      if (!(atomicOr(&m.fin[sl >> 5], bit) & bit)) {
        const uint32_t p = atomicAdd(&sh.nn[1], 1u);
        if (p < cp.F) m.front0[p] = (uint16_t)sl;
      }
    }
    for (uint32_t j = tid; j < nc0 && j < cp.C; j += T) {
      const unsigned long long a = __ldcg(rv.cand + j);
      const uint32_t s0 = (uint32_t)(a >> 32);
      int ns = (int)SPECIAL;
      if (s0 != SPECIAL) {
        ns = tab_find(m, H, __ldcg(rv.key + s0));
        if (ns < 0) atomicOr(&sh.flags, FL_OVF);
      }
      m.cand[j] = ((unsigned long long)(uint32_t)ns << 32) | (uint32_t)a;
      m.cobj[j] = __ldcg(rv.cobj + j);
    }
    if (tid == 0) {
      sh.nc = nc0;
      rmask |= __ldcg(&rv.hdr->rmask);
      atomicAdd(&s.st->ex_resumed, 1ull);
    }
    __syncthreads();
    nf = sh.nn[1];
    if (nf > cp.F || nc0 > cp.C || (sh.flags & FL_OVF)) return OVERFLOW;
    uint32_t mn = INF;
    for (uint32_t i = tid; i < nf; i += T) mn = min(mn, DISTR(m, m.front0[i]));
    mn = __reduce_min_sync(FULL, mn);
    if (lane == 0) sh.red[1][wid] = mn;
    __syncthreads();
    blo = sh.red[1][0];
#pragma unroll
    for (int w = 1; w < W; ++w) blo = min(blo, sh.red[1][w]);
    // (sh.nn[1] and sh.red[1] are round 1's: round 0 resets nn[1] after its bucket barrier,
    // which every thread passes after reading nf above)
  } else {
    if (tid == 0) {
      const uint32_t seed_v = q.y == 0 ? ei.x : g.edst[q.x];
      bool imp;
      const int sl = tab_relax(m, H, seed_v, seed_d, imp);
      m.front0[0] = (uint32_t)sl;
      m.fin[sl >> 5] |= 1u << (sl & 31);
    }
    // objects on q's own arc ahead of q (reading R2), stored at vertex src(q.e)
    if (q.y > 0) {
      const uint32_t c = cellof(g, ei.x);
      if (s.cell_head[c] != NONE) {
        if (tid == 0) request_flush(s, c, P.epoch);
        return RETRY;
      }
      const uint2 vo = vobj_valid(s.v_obj[ei.x], s.cell_comp[c]);
      for (uint32_t j = tid; j < vo.y; j += T) {
        const uint32_t p = vo.x + j;
        const uint32_t ob = s.ar.obj[p];
        const uint32_t oe = s.ar.edge[p], oo = s.ar.off[p];
        if (oe == q.x && oo >= q.y && valid_rec(s, p, ob)) {
          const uint32_t i = atomicAdd(&sh.nc, 1u);
          if (i < cp.C) {
            m.cand[i] = ((unsigned long long)SPECIAL << 32) | (oo - q.y);
            m.cobj[i] = ob;
          }
        }
      }
    }
    __syncthreads();
    if (sh.nc > cp.C) return OVERFLOW;
  }

  auto* front = m.front0;
  auto* nfront = m.front1;
  // frontier size and minimum: the next frontier holds the re-queued entries (their D read at
  // partition) and every vertex improved during the round (each improvement's new D is seen
  // here), so the minimum over those is exact
  uint32_t c_iter = 0, c_vert = 0, c_arcs = 0, c_harv = 0, c_objs = 0;
  for (uint32_t rnd = 0;; ++rnd) {
    const uint32_t par = rnd & 1;
    ++c_iter;
    // ---- 1. termination (nf, blo and the candidates are the same for every thread)
    if (nf == 0 || blo > lim) break;
    // warp 0 counts the candidates; the others partition meanwhile and read the verdict
    // after the bucket barrier (a stopping round's partition is simply dropped)
    const uint32_t nc0 = sh.nc;
    if (nc0 >= k && wid == 0) {
      uint32_t cl = 0;
      for (uint32_t i = lane; i < nc0; i += 32) cl += cand_dist(m, i) < blo;
      if (__reduce_add_sync(FULL, cl) >= k && lane == 0) sh.stop[par] = 1;
    }
    // ---- 2. partition the frontier: the bucket [m, m + delta) is expanded, the rest re-queued
    const uint32_t bhi = (blo > INF - g.delta) ? INF : blo + g.delta;
    uint32_t mn = INF;
    for (uint32_t i = tid; i < nf; i += T) {
      const uint32_t sl = front[i];
      const uint32_t ent = DISTR(m, sl);
      if (ent < bhi) {
        m.act[atomicAdd(&sh.na[par], 1u)] = sl;  // (act has F entries: na <= nf <= F)
        atomicAnd(&m.fin[sl >> 5], ~(1u << (sl & 31)));
      } else {
        nfront[atomicAdd(&sh.nn[par], 1u)] = sl;
        mn = min(mn, ent);
      }
    }
    __syncthreads();  // the bucket is complete
    if (sh.stop[par]) break;
    const uint32_t na = sh.na[par];
    if (tid == 0) {  // the next round's counters (their last readers are past the barrier)
      sh.nn[par ^ 1] = 0;
      sh.na[par ^ 1] = 0;
      sh.stop[par ^ 1] = 0;
      c_vert += na;
    }
    // ---- 3. expand: lane = (vertex, arc slot), T/4 vertices per window; no barrier between
    //         windows (appends and candidates are reserved with shared atomics; the outcome
    //         flags are read at the end of the round)
    for (uint32_t w0 = 0; w0 < na; w0 += T / 4) {
      const uint32_t vi = w0 + (tid >> 2), s4 = tid & 3;
      if (vi < na) {
        const uint32_t vslot = m.act[vi];
        const uint32_t u = KEYR(m, vslot), du = DISTR(m, vslot);  // D re-read after the frontier bit
        const uint2 arc = g.vadj[(size_t)u * 4 + s4];
        bool harv = false;
        uint32_t hcell = 0, hd = NONE;
        uint2 cc = make_uint2(0, 0), v0 = make_uint2(0, 0);
        if (s4 == 0) {
          hcell = cellof(g, u);
          hd = s.cell_head[hcell];
          cc = s.cell_comp[hcell];
          if (!GG_VHAS || vhas_bit(s, u)) v0 = s.v_obj[u];
          harv = !(atomicOr(&m.listed[vslot >> 5], 1u << (vslot & 31)) & (1u << (vslot & 31)));
        }
        auto relax = [&](uint32_t dst, uint32_t w) {
          ++c_arcs;
          const unsigned long long nd = (unsigned long long)du + w;
          if (nd >= INF) return;
          bool imp;
          const int rr = tab_relax(m, H, dst, (uint32_t)nd, imp);
          if (rr < 0) {
            atomicOr(&sh.flags, FL_OVF);
          } else if (imp) {
            mn = min(mn, (uint32_t)nd);
            const uint32_t bit = 1u << (rr & 31);
            if (!(atomicOr(&m.fin[rr >> 5], bit) & bit)) {
              prefetch_vertex(g, s, dst);
              const uint32_t p = atomicAdd(&sh.nn[par], 1u);
              if (p < cp.F) nfront[p] = (uint32_t)rr;
              else atomicOr(&sh.flags, FL_OVF);
            }
          }
        };
        if (arc.y == WMAX) {  // more than 4 arcs: slot 3 continues in the CSR
          for (uint32_t a = g.rowptr[u] + 3; a < g.rowptr[u + 1]; ++a) {
            const uint2 av = g.adj[a];
            relax(av.x, av.y);
          }
        } else if (arc.y != 0) {
          relax(arc.x, arc.y);
        }
        if (harv) {
          ++c_harv;
          if (track) {
            const uint32_t o = owner_of(hcell, g.n_cells, s.n_ranks);
            if (o != s.rank) rmask |= 1ull << o;
          }
          if (hd != NONE) {  // cached updates: lazy flush, then retry
            request_flush(s, hcell, P.epoch);
            atomicOr(&sh.flags, FL_RETRY);
          } else {
            const uint2 vo = vobj_valid(v0, cc);
            c_objs += vo.y;
            for (uint32_t j = 0; j < vo.y; ++j) {
              const uint32_t p = vo.x + j;
              const uint32_t ob = s.ar.obj[p];
              const unsigned long long kk = s.ar.key[p];
              const uint32_t oe = s.ar.edge[p], oo = s.ar.off[p];
              const bool same_ahead = q.y > 0 && oe == q.x && oo >= q.y;  // already a candidate
              if (!same_ahead && (!GG_HARVEST_VALIDATE || kk == s.ot_key[ob])) {
                const uint32_t i = atomicAdd(&sh.nc, 1u);
                if (i < cp.C) {
                  m.cand[i] = ((unsigned long long)vslot << 32) | oo;
                  m.cobj[i] = ob;
                } else {
                  atomicOr(&sh.flags, FL_OVF);
                }
              }
            }
          }
        }
      }
    }
    // ---- 4. round complete: the next frontier's minimum, the outcome flags
    mn = __reduce_min_sync(FULL, mn);
    if (lane == 0) sh.red[par][wid] = mn;
    __syncthreads();
    const uint32_t fl = sh.flags;
    if (fl & FL_OVF) return OVERFLOW;
    if (fl & FL_RETRY) {  // ask for every dirty cell the frontier will need, then retry
      for (uint32_t i = tid; i < nf; i += T) request_flush(s, cellof(g, KEYR(m, front[i])), P.epoch);
      return RETRY;
    }
    blo = sh.red[par][0];
#pragma unroll
    for (int w = 1; w < W; ++w) blo = min(blo, sh.red[par][w]);
    nf = sh.nn[par];
    auto* tmp = front;
    front = nfront;
    nfront = tmp;
  }

  // every warp leaves the loop in the same round (the verdicts are read after barriers); this
  // barrier keeps a warp from rewriting the candidates below before every warp has left
  __syncthreads();
  // the k smallest (dist, obj)
  const uint32_t nc = sh.nc;
  for (uint32_t i = tid; i < nc; i += T) {
    const unsigned long long d = cand_dist(m, i);
    m.cand[i] = d < INF ? ((d << 32) | m.cobj[i]) : EMPTY64;
  }
  __syncthreads();
  block_sort<W>(m.cand, nc, cp.C);
  for (uint32_t r = tid; r < k; r += T) {
    const unsigned long long dk = r < nc ? m.cand[r] : EMPTY64;
    const bool ok = dk != EMPTY64 && (uint32_t)(dk >> 32) <= lim;
    P.out_obj[(size_t)qi * k + r] = ok ? (uint32_t)dk : GGRID_PAD;
    P.out_dist[(size_t)qi * k + r] = ok ? (uint32_t)(dk >> 32) : GGRID_PAD;
  }
  if (P.remote) {
    unsigned long long x = rmask;
    x = ((unsigned long long)__reduce_or_sync(FULL, (uint32_t)(x >> 32)) << 32) |
        __reduce_or_sync(FULL, (uint32_t)x);
    if (lane == 0) sh.redl[wid] = x;
    __syncthreads();
    if (tid == 0) {
      unsigned long long r = 0;
      for (int w = 0; w < W; ++w) r |= sh.redl[w];
      P.remote[qi] = r;
    }
  }
  const uint32_t sa = block_sum<W>(c_arcs, sh), sh_ = block_sum<W>(c_harv, sh), so = block_sum<W>(c_objs, sh);
#if GG_TAIL_DEBUG
  if (tid == 0 && P.level > 0) printf("W %u %u %u %u\n", qi, c_iter, c_vert, sa);
#endif
  if (tid == 0) {
    atomicAdd(&s.st->ex_iters, (unsigned long long)c_iter);
    atomicAdd(&s.st->ex_vertices, (unsigned long long)c_vert);
    atomicAdd(&s.st->ex_arcs, (unsigned long long)sa);
    atomicAdd(&s.st->ex_harvested, (unsigned long long)sh_);
    atomicAdd(&s.st->ex_objects, (unsigned long long)so);
  }
  __syncthreads();
  return DONE;
}

// warps per query of the CTA variant: 4 at the starting level (the bench's balls of ~300
// vertices, ~17 per round: one window of 32 vertices per round; measured 4 > 3 > 5 > 2 > 6 > 8
// warps per query, and one warp per query slower than all but 8), 8 at the larger levels
// (experiment hooks).  ptxas fits the 4-warp kernel in 32 registers (a few bytes of spills),
// i.e. 16 CTAs = 64 warps per SM; capping it at 40-56 registers (launch-bounds min blocks
// 12-1) measured 8-23% slower.
#ifndef GG_CTA_W0
#define GG_CTA_W0 4
#endif
#ifndef GG_CTA_W
#define GG_CTA_W 8
#endif
constexpr int CTA_W0 = GG_CTA_W0, CTA_W = GG_CTA_W;
__host__ __device__ constexpr int cta_warps(int level) { return level <= 1 ? CTA_W0 : CTA_W; }
#ifndef GG_CTA_LEVEL
#define GG_CTA_LEVEL 0  // first level run CTA-per-query (experiment hook; 1: level 0 one warp per query)
#endif

// resident CTAs per SM asked of ptxas (a register cap: 40) for the fixed-capacity level (level
// 1; measured at C2 k=50: 0.496 ms vs 0.575 at 32 registers and 0.545 with runtime capacities).
// Level 0 keeps runtime capacities: ptxas's own choice there (32 registers, 16 CTAs) measured
// 3% faster at C1 than either fixed-capacity build.
#ifndef GG_MINB0
#define GG_MINB0 12
#endif
template <int W, class CP>
__device__ __forceinline__ void expand_cta_body(const QParams& P) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ CtaShared<W> sh;
  __shared__ uint32_t qslot, rslot;
  const WarpMemS m = carve<uint16_t>(smem_raw, CP::get(P));
  pdl_trigger(P);
  for (;;) {  // persistent: queries fetched dynamically
    if (threadIdx.x == 0) {
      const uint32_t li = atomicAdd(&P.s.st->expand_work[P.level], 1u);
      uint32_t qi = NONE;
      rslot = NONE;
      if (li < P.n) {
        qi = P.qlist ? P.qlist[li] : li;
      } else if (P.chain_in && li - P.n < P.chain_cap) {
        // a chained level running beside the level below: take the next promoted query as
        // soon as it is written, until every CTA below has exited (promotions published)
        volatile uint32_t* slot = P.chain_in + (li - P.n);
        for (;;) {
          uint32_t v = *slot;
          if (v == NONE && *(volatile const uint32_t*)P.wait_exited == P.wait_total) {
            __threadfence();
            v = *slot;
            if (v == NONE) break;
          }
          if (v != NONE) {
            qi = v;
            *slot = NONE;  // (the ring is all-NONE again when the level has drained it)
            if (P.resume && li - P.n < P.resume_cap) {
              __threadfence();  // (the record was written before the entry)
              rslot = li - P.n;
            }
            break;
          }
          __nanosleep(1000);
        }
      }
      qslot = qi;
    }
    __syncthreads();
    const uint32_t qi = qslot, rs = rslot;
    __syncthreads();
    if (qi == NONE) break;
#if GG_TAIL_DEBUG
    const unsigned long long t0 = gtime();
#endif
    const int r = run_query_cta<W, CP>(P, m, sh, qi, rs);
    if (threadIdx.x == 0 && r != DONE) finish_undone(P, qi, r);
#if GG_TAIL_DEBUG
    if (threadIdx.x == 0 && P.level > 0) printf("L %u %d %llu %llu\n", qi, r, t0, gtime());
#endif
    __syncthreads();
  }
  if (threadIdx.x == 0) count_exit(P);
}
// (two kernels: an explicit min-blocks launch bound changes ptxas's register choice even at 1)
template <int W, class CP>
__global__ void __launch_bounds__(W * 32) k_expand_cta(QParams P) {
  expand_cta_body<W, CP>(P);
}
template <int W, class CP>
__global__ void __launch_bounds__(W * 32, GG_MINB0) k_expand_cta_capped(QParams P) {
  expand_cta_body<W, CP>(P);
}

// Capacity ladder.  Levels 0-5 keep the query's working set in shared memory (~11, 15, 28, 45,
// 95 and 190 KB): level 0 one warp per query when small balls are expected (as many
// single-warp CTAs per SM as fit), else, like levels 1-5, one CTA per query (k_expand_cta: 4
// warps at levels 0-1, 8 above); level 6 is global memory sized from |V| (a query that reaches
// fewer than k objects may need to settle the whole graph).
constexpr int NLEVELS = EXPAND_LEVELS;
#ifndef GG_H0
#define GG_H0 1024  // level-0 vertex table of the CTA-per-query kernel (experiment hook: -DGG_H0=...)
#endif
// ... and of the one-warp-per-query kernel (small expected balls, C3): fewer slots = more queries
// resident per SM (with 4 warps per CTA: 1,024 -> 896 -> 768 slots = 18 -> 20 -> 24 warps per SM;
// C3 expansion 1.66 -> 1.46 -> 1.37 ms, 7 promotions per 65,536 queries at 768)
// the one-warp level 0's frontier and candidate capacities (C3 replay of 1,000 queries: frontier
// <= 57, harvested candidates <= 16 at k = 10); k above GG_C0W - 32 starts at the CTA kernel.
// Measured at C3 (r2 A/B): 32 resident queries per SM (696 slots, 64-entry stage with the half
// split, F 64, C 32: 7,024 B, 64 registers with spills) 1.146 ms vs 1.115 ms for this 28-resident
// configuration; without the half split 71% of the queries promote (chunks of > 64 arcs)
#ifndef GG_F0W
#define GG_F0W 64
#endif
#ifndef GG_C0W
#define GG_C0W 64
#endif
static_assert((GG_C0W & (GG_C0W - 1)) == 0, "the candidate list is bitonic-sorted: a power of two");
#ifndef GG_H0W
#define GG_H0W 600
#endif
#ifndef GG_F0
#define GG_F0 96
#endif
#ifndef GG_C0
#define GG_C0 64
#endif
// level 1 takes 32 < k <= 96 (measured C2 k=40: 0.47 ms there vs 0.68 ms at the 2048-slot level;
// widening level 0's candidate list instead cost the k=10 configs 2-4%).  Candidate capacities
// are powers of two: the bitonic sorts pad to one.
using Caps0 = FixCaps<GG_H0, GG_F0, GG_C0>;
using Caps1 = FixCaps<1280, 128, 128>;
const Caps kCaps[NLEVELS - 1] = {Caps0::caps(),     Caps1::caps(),     {2048, 512, 256},
                                 {4096, 1024, 256}, {8192, 2048, 512}, {16384, 4096, 2048}};

// the CTA kernel of a shared-memory level
using CtaKernel = void (*)(QParams);
static CtaKernel cta_kernel(int level) {
  if (level == 0) return k_expand_cta<CTA_W0, DynCaps>;
  if (level == 1) return k_expand_cta_capped<CTA_W0, Caps1>;
  return k_expand_cta<CTA_W, DynCaps>;
}

Caps caps_for(int level, uint32_t V) {
  if (level < NLEVELS - 1) return kCaps[level];  // (level 0 one-warp mode: caps_mode below)
  uint32_t H = 1u << 15;
  while (H < 2ull * V && H < (1u << 27)) H <<= 1;
  const uint32_t F = std::min<uint32_t>(H / 2, 1u << 22);
  return Caps{H, F, 8192};
}

}  // namespace

int expand_levels() { return NLEVELS; }

uint32_t expand_table_slots(int level) { return caps_for(level, 1).H; }

uint32_t expand_max_k(int level) { return caps_for(level, 1).C - 32; }

// The one-warp level 0 has two tables: the narrow one (600 slots, frontier 64: 7,008 B per query,
// 32 queries per SM) and, when the caller's hint says the expected ball touches more vertices
// (WIDE_BIT of ball_hint: expected ball x arcs per vertex above ~650, e.g. C1's denser NY-shaped
// graph), the wide one (704 slots, frontier 96: 28 per SM).  Measured: C3 expansion 1.030 ->
// 0.986 ms narrow; C1 0.262 ms wide vs 0.360 narrow; C2 k=30 0.268 wide vs 0.286 narrow.
#ifndef GG_H0W_WIDE
#define GG_H0W_WIDE 704
#endif
#ifndef GG_F0W_WIDE
#define GG_F0W_WIDE 96
#endif
// SMALLK_BIT (k <= 16 with the narrow table): a 32-entry candidate list buys 48 more slots (648)
// at the same 32 resident queries per SM (C3: 0.988 -> 0.979 ms)
#ifndef GG_H0W_SMALLK
#define GG_H0W_SMALLK 648
#endif
constexpr uint32_t WIDE_BIT = 1u << 31, SMALLK_BIT = 1u << 30;
__host__ __device__ inline bool wide0(uint32_t bh) { return (bh & WIDE_BIT) != 0; }
// table variant of the one-warp level 0: 0 narrow, 1 wide, 2 narrow with the short candidate list
__host__ __device__ inline int var0(uint32_t bh) { return (bh & WIDE_BIT) ? 1 : (bh & SMALLK_BIT) ? 2 : 0; }
__host__ __device__ inline uint32_t ball_of(uint32_t bh) { return bh & ~(WIDE_BIT | SMALLK_BIT); }
// the caps a level runs with in a given mode (the one-warp kernel's level 0 has its own tables)
static Caps caps_mode(int level, uint32_t V, bool cta, int var = 0) {
  Caps c = caps_for(level, V);
  if (level == 0 && !cta) {
    c.H = var == 1 ? GG_H0W_WIDE : var == 2 ? GG_H0W_SMALLK : GG_H0W;
    c.F = var == 1 ? GG_F0W_WIDE : GG_F0W;
    c.C = var == 2 ? 32u : (uint32_t)GG_C0W;
  }
  return c;
}
static size_t warp_bytes_mode(int level, uint32_t V, bool cta, int var = 0) {
  return (warpmem_bytes(caps_mode(level, V, cta, var), level == NLEVELS - 1 ? 4 : 2) + 15) & ~size_t(15);
}

size_t expand_warp_bytes(int level, uint32_t V) {
  const Caps c = caps_for(level, V);
  return (warpmem_bytes(c, level == NLEVELS - 1 ? 4 : 2) + 15) & ~size_t(15);
}

// CTA-per-query for the shared-memory levels, and for small batches at any of them; the
// starting level runs one warp per query when the caller expects small balls (ball_hint below
// kCtaBall vertices: measured C2 k=10, ball ~110: one warp 0.179 ms vs 4 warps 0.194 ms; C3,
// ~240: 36.9 vs 36.3M q/s; C1, ~260: 0.330 vs 0.273 ms; C2 k=30, ~320: 0.398 vs 0.345 ms)
// (with the bucketed table, r2: C1 expansion 0.301 -> 0.262 ms and C2 k=30 0.370 -> 0.268 ms one
// warp per query; thresholds 400 and 600 equal on both, so 512)
#ifndef GG_CTA_BALL
#define GG_CTA_BALL 512
#endif
#ifndef GG_CTA_BALL1
#define GG_CTA_BALL1 1024  // (C2 k=40 / 50: expansion 0.427 -> 0.401 / 0.489 -> 0.474 ms; 0: always a CTA)
#endif
constexpr uint32_t kCtaBall = GG_CTA_BALL;
#ifndef GG_WARP_MAXK
#define GG_WARP_MAXK (GG_C0W - 32)
#endif
uint32_t expand_warp_max_k() { return GG_WARP_MAXK; }
uint32_t expand_cta_ball() { return kCtaBall; }
static bool use_cta(int level, uint32_t n, int sm_count, uint32_t ball_hint) {
  ball_hint = ball_of(ball_hint);
  if (level >= NLEVELS - 1) return false;
  if (n <= (uint32_t)sm_count) return true;
  if (level == 0) return GG_CTA_LEVEL == 0 && ball_hint >= kCtaBall;
  // (a starting level 1 -- 32 < k <= 96 -- also runs one warp per query below GG_CTA_BALL1)
  if (level == 1) return ball_hint >= GG_CTA_BALL1;
  return true;
}

// bytes of one resumable-promotion record when `level` starts a batch of n queries with the
// one-warp kernel (which exports the state of the queries it promotes), else 0
size_t expand_resume_bytes(int level, uint32_t n, int sm_count, uint32_t ball_hint) {
  if (level >= NLEVELS - 2 || use_cta(level, n, sm_count, ball_hint) || (GG_PAIR && level == 0)) return 0;
  return resume_bytes(caps_mode(level, 1, false, var0(ball_hint)));
}

// one-warp-per-query kernel: warps (independent queries) per CTA.  Each CTA costs 1 KB of reserved
// shared memory beside its warps' tables, so several warps per CTA fit more queries per SM
#ifndef GG_WARP_WPC
#define GG_WARP_WPC 4
#endif
constexpr uint32_t WPC = GG_WARP_WPC;

// resident CTAs per SM of a shared-memory level's kernel (occupancy calculator, cached)
static uint32_t blocks_per_sm(int level, bool cta, int var = 0) {
  static int bps[3][2][NLEVELS] = {};  // (occupancy: the same on every B200)
  // the attribute is per device: set on every device this process launches on
  if (cta) func_attr_once(cta_kernel(level), cudaFuncAttributeMaxDynamicSharedMemorySize, 226 * 1024);
  else if (GG_PAIR && level == 0) func_attr_once(k_expand_pair, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
  else func_attr_once(k_expand<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
  int& b = bps[var][cta ? 1 : 0][level];
  if (!b) {
    const int smem = (int)warp_bytes_mode(level, 1, cta, var);
    if (cta) {
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, cta_kernel(level), cta_warps(level) * 32, smem);
    } else {
      if (GG_PAIR && level == 0)  // (two queries per warp: two tables per warp)
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_expand_pair, 32 * WPC, 2 * smem * WPC);
      else
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_expand<true>, 32 * WPC, smem * WPC);
    }
#ifdef GG_L0_PER_SM
    if (!cta && level == 0) b = std::min(b, GG_L0_PER_SM);  // experiment hook: occupancy cap
#endif
    if (b <= 0) b = 1;
  }
  return (uint32_t)b;
}

uint32_t expand_grid(int level, uint32_t n, int sm_count, uint32_t ball_hint) {
  if (level == NLEVELS - 1) return 0;  // (global scratch: sized by the caller's scratch warps)
  const bool cta = use_cta(level, n, sm_count, ball_hint);
  const uint32_t per = cta ? 1u : (GG_PAIR && level == 0 ? 2 * WPC : WPC);  // queries a CTA runs at once
  return std::min<uint32_t>((n + per - 1) / per, (uint32_t)sm_count * blocks_per_sm(level, cta, var0(ball_hint)));
}

size_t expand_block_bytes(int level, uint32_t V, uint32_t n, int sm_count, uint32_t ball_hint, bool chained) {
  if (level == NLEVELS - 1) return 0;
  const bool cta = chained || use_cta(level, n, sm_count, ball_hint);
  const uint32_t per = cta ? 1u : (GG_PAIR && level == 0 ? 2 * WPC : WPC);
  return warp_bytes_mode(level, V, cta, var0(ball_hint)) * per + 1024;  // (+ the per-CTA reservation)
}

void launch_expand(const ExpandLaunch& L, const DevGraph& g, const DevState& s, int sm_count, cudaStream_t st) {
  const int level = L.level;
  if (L.n == 0 && !L.chain_in) return;
  QParams P;
  P.g = g;
  P.s = s;
  P.q = L.q;
  P.qlist = L.qlist;
  P.n = L.n;
  P.k = L.k;
  P.epoch = L.epoch;
  P.level = level;
  P.last_level = NLEVELS - 1;
  P.retry_list = L.retry_list;
  P.promote_list = L.promote_list;
  P.promote_count = L.promote_count;
  P.out_obj = L.out_obj;
  P.out_dist = L.out_dist;
  P.bound = L.bound;
  P.remote = L.remote;
  const bool cta_mode = level < NLEVELS - 1 && (L.chain_in != nullptr || use_cta(level, L.n, sm_count, L.ball_hint));
  const int var = var0(L.ball_hint);
  P.caps = caps_mode(level, g.V, cta_mode, var);
  P.warps_per_cta = 1;  // (the one-warp shared-memory kernel: WPC, set below)
  P.scratch = nullptr;
  P.exited = L.exited;
  P.chain_in = const_cast<uint32_t*>(L.chain_in);
  P.chain_cap = L.chain_cap;
  P.wait_exited = L.wait_exited;
  P.wait_total = L.wait_total;
  P.trigger = L.trigger ? 1 : 0;
  P.wait_prior = L.chain_in ? 0 : 1;  // (a chained level runs beside the level below it)
  P.resume = nullptr;
  P.resume_cap = 0;
  P.resume_bytes = 0;
  P.rcaps = Caps{0, 0, 0};
  if (L.resume && L.resume_cap) {  // (the exporting level: this one, or the one below a chained level)
    P.rcaps = caps_mode(L.chain_in ? level - 1 : level, g.V, false, var);
    P.resume = static_cast<unsigned char*>(L.resume);
    P.resume_cap = L.resume_cap;
    P.resume_bytes = (uint32_t)resume_bytes(P.rcaps);
  }
  const int smem = (int)warp_bytes_mode(level, g.V, cta_mode, var);
  if (level == NLEVELS - 1) {
    P.scratch = static_cast<unsigned char*>(L.scratch);
    k_expand<false><<<std::min<uint32_t>(L.n, std::max<uint32_t>(1, L.scratch_warps)), 32, 0, st>>>(P);
    return;
  }
  const bool cta = L.chain_in != nullptr || use_cta(level, L.n, sm_count, L.ball_hint);
  const uint32_t grid = L.grid ? L.grid : std::max<uint32_t>(1, expand_grid(level, L.n, sm_count, L.ball_hint));
  blocks_per_sm(level, cta, var);  // (sets the shared-memory attribute)
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  const bool pair = !cta && GG_PAIR && level == 0;
  if (!cta) P.warps_per_cta = WPC;
  cfg.blockDim = dim3(cta ? cta_warps(level) * 32 : 32 * WPC);
  cfg.dynamicSmemBytes = (size_t)smem * (cta ? 1 : (pair ? 2 * WPC : WPC));
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;  // programmatic dependent of the flush (waits for it) or, chained, of the level below
  if (cta) {
    cudaLaunchKernelEx(&cfg, cta_kernel(level), P);
  } else if (pair) {
    cudaLaunchKernelEx(&cfg, k_expand_pair, P);
  } else {
    cudaLaunchKernelEx(&cfg, k_expand<true>, P);
  }
}

}  // namespace gg

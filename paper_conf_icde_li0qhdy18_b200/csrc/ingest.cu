// ingest.cu — caching location-update messages (Alg. 1, P@18177-19248) on the device.
//
// The paper appends each message to the bucket list of cell getCell(m.e) on the CPU,
// appends a tombstone to the old cell and overwrites the object table (Alg. 1).  Here a
// batch of n updates becomes, in three launches:
//   classify : validate, find cell(src(e)) via the inverted index (P@15006), warp-
//              aggregated rank within the cell (one atomic per distinct cell per warp);
//   alloc    : one thread per cell carves this batch's extent for the cell out of the
//              bump arena (warp-aggregated) and links it at the head of the cell's chain;
//   scatter  : writes the SoA record and RED.MAX-es (t<<32|seq) into ot_key[o].
// A batch that fits one resident wave runs the same three phases as ONE cooperative launch
// with grid barriers between them: k_ingest_fused (per-tile cell hash in shared memory, for
// batches with many updates per distinct cell) or k_ingest_direct (one rank atomic per
// update, state in registers, for batches spread over many more cells than a tile holds).
// No tombstones: a record is valid iff its key equals ot_key[obj] (reading R8/R9), which
// also makes out-of-order arrivals harmless.
#include <algorithm>
#include <cstdio>

#include "internal.cuh"

namespace gg {

// CTA-level aggregation: each CTA takes CU consecutive updates (a tile), counts them per cell
// in a shared-memory hash (rank within the CTA), then claims one global range per distinct
// cell with a single atomicAdd on bcount[cell] (few cells => no hot-spot serialisation).
// It also orders its tile by cell (hash slot): tmp[] holds, in that order, each update's
// (source vertex, rank in the cell's batch extent) and perm[] its index in the tile, so the
// scatter's consecutive threads write consecutive arena positions (runs per cell).
#ifndef GG_INGEST_CT
#define GG_INGEST_CT 1024
#endif
constexpr int CT = GG_INGEST_CT;   // threads
#ifndef GG_INGEST_CPT
#define GG_INGEST_CPT 8
#endif
constexpr int CPT = GG_INGEST_CPT; // updates per thread
constexpr int CU = CT * CPT;       // updates per CTA (tile)
constexpr int CH = 2 * CU;         // hash slots (>= 2*CU)
constexpr int CH_BITS = 31 - __builtin_clz(CH);
static_assert((1 << CH_BITS) == CH, "hash slots: a power of two");
constexpr int SPC = CH / CT;       // hash slots per thread in the scan
constexpr int SCATTER_SMEM = CU * 16;
static_assert(CU < 65536, "tile offsets and counts are packed in 16 bits");
static_assert(CPT % 2 == 0, "the scatter works in two halves of CPT/2 updates per thread");
constexpr uint32_t REMOTE_CELL = 0xFFFFFFFEu;  // classify: pseudo-cell of other ranks' updates
constexpr int CLASSIFY_SMEM = (3 * CH + CT / 32) * 4;
static_assert(CLASSIFY_SMEM <= 227 * 1024, "classify tile state exceeds shared memory");
static_assert(SCATTER_SMEM <= 227 * 1024, "scatter tile exceeds shared memory");

__global__ void __launch_bounds__(CT) k_ingest_classify(const uint4* __restrict__ upd, uint64_t n,
                                                        DevGraph g, DevState s,
                                                        uint2* __restrict__ tmp,
                                                        uint16_t* __restrict__ perm) {
  extern __shared__ __align__(16) uint32_t h_buf[];  // CLASSIFY_SMEM bytes
  uint32_t* h_cell = h_buf;           // cell id; after the claim, the cell's global rank base
  uint32_t* h_cnt = h_buf + CH;       // count; after the scan, (tile offset << 16) | count
  uint32_t* h_tmax = h_buf + 2 * CH;  // newest t per cell (the extent's zeta.t)
  uint32_t* w_sum = h_buf + 3 * CH;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  for (int i = tid; i < CH; i += CT) {
    h_cell[i] = NONE;
    h_cnt[i] = 0;
    h_tmax[i] = 0;
  }
  __syncthreads();
  const uint64_t base = (uint64_t)blockIdx.x * CU;
  uint32_t tl = 0;  // this thread's newest t
  int slot[CPT];
  uint32_t vs[CPT], lr[CPT];
  // all CPT record loads in flight, then all CPT inverted-index gathers, then the hashing
  uint4 mm[CPT];
#pragma unroll
  for (int j = 0; j < CPT; ++j) {
    const uint64_t i = base + (uint64_t)j * CT + tid;
    mm[j] = i < n ? __ldg(upd + i) : make_uint4(0, 0xFFFFFFFFu, 0, 0);  // re-read by scatter
  }
  uint2 ee[CPT];
#pragma unroll
  for (int j = 0; j < CPT; ++j) ee[j] = mm[j].y < g.A ? __ldg(g.einfo + mm[j].y) : make_uint2(0, 1);
#pragma unroll
  for (int j = 0; j < CPT; ++j) {
    const uint64_t i = base + (uint64_t)j * CT + tid;
    slot[j] = -1;
    if (i >= n) continue;
    const uint4 m = mm[j];
    const uint2 e = ee[j];
    unsigned bad = 0;
    if (m.x >= s.max_objects) bad |= ERR_OBJ;
    if (m.y >= g.A) {
      bad |= ERR_EDGE;
    } else if (m.z >= e.y) {
      bad |= ERR_OFF;
    }
    if (bad) {
      atomicOr(&s.st->ingest_err, bad);
      atomicMin(&s.st->bad_index, i < 0xFFFFFFFFull ? (unsigned)i : 0xFFFFFFFFu);
      continue;
    }
    // updates of cells another rank owns (sharded mode) are grouped under one pseudo-cell:
    // no record here, only the object-table update (in the scatter, after validation)
    const uint32_t c0 = cellof(g, e.x);
    const bool remote = s.n_ranks > 1 && owner_of(c0, g.n_cells, s.n_ranks) != s.rank;
    const uint32_t c = remote ? REMOTE_CELL : c0;
    uint32_t h = (c * 2654435761u) >> (32 - CH_BITS);
    volatile uint32_t* vc = h_cell;
    for (;;) {
      const uint32_t cur = vc[h];
      if (cur == c) break;
      if (cur == NONE) {
        const uint32_t old = atomicCAS(&h_cell[h], NONE, c);
        if (old == NONE || old == c) break;
      }
      h = (h + 1) & (CH - 1);
    }
    slot[j] = (int)h;
    vs[j] = e.x;
    lr[j] = atomicAdd(&h_cnt[h], 1u);
    atomicMax(&h_tmax[h], m.w);
    tl = max(tl, m.w);
  }
  tl = __reduce_max_sync(0xffffffffu, tl);
  if (lane == 0 && tl) atomicMax(&s.st->batch_tmax, tl);  // (t_max: only if accepted, k_ingest_alloc)
  __syncthreads();
  // exclusive scan of the slot counts = each cell's group offset in the tile's sorted order
  {
    uint32_t loc[SPC], sum = 0;
#pragma unroll
    for (int q = 0; q < SPC; ++q) {
      loc[q] = sum;
      sum += h_cnt[tid * SPC + q];
    }
    uint32_t x = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) w_sum[wid] = x;
    __syncthreads();
    uint32_t wpre = 0;
    for (int w = 0; w < wid; ++w) wpre += w_sum[w];
    const uint32_t excl = wpre + x - sum;
#pragma unroll
    for (int q = 0; q < SPC; ++q) h_cnt[tid * SPC + q] |= (excl + loc[q]) << 16;  // counts <= CU
  }
  __syncthreads();  // (the claims below read other threads' slots)
  {  // one claim per distinct cell of the tile: all of a thread's SPC returning atomics in flight
     // together (a loop storing each result before the next load serialises their latencies)
    uint32_t cs[SPC], base[SPC];
#pragma unroll
    for (int q = 0; q < SPC; ++q) cs[q] = h_cell[q * CT + tid];
#pragma unroll
    for (int q = 0; q < SPC; ++q) {
      const uint32_t c = cs[q], i = q * CT + tid;
      base[q] = c;
      if (c != NONE && c != REMOTE_CELL) {
        atomicMax(&s.bcount[c * BCOUNT_STRIDE + 1], h_tmax[i]);
        base[q] = atomicAdd(&s.bcount[c * BCOUNT_STRIDE], h_cnt[i] & 0xFFFFu);
      }
    }
#pragma unroll
    for (int q = 0; q < SPC; ++q) h_cell[q * CT + tid] = base[q];
  }
  __syncthreads();
  uint32_t si[CPT], rk[CPT];
#pragma unroll
  for (int j = 0; j < CPT; ++j) {
    if (slot[j] < 0) continue;
    si[j] = (h_cnt[slot[j]] >> 16) + lr[j];
    rk[j] = h_cell[slot[j]] == REMOTE_CELL ? NONE : h_cell[slot[j]] + lr[j];
  }
  __syncthreads();
  // the tile in cell order, staged in the (now free) hash table, then written coalesced
  uint2* stg = reinterpret_cast<uint2*>(h_buf);            // CU x 8 B
  uint16_t* stp = reinterpret_cast<uint16_t*>(h_buf + CH);  // CU x 2 B
#pragma unroll
  for (int j = 0; j < CPT; ++j) {
    if (slot[j] < 0) continue;
    stg[si[j]] = make_uint2(vs[j], rk[j]);
    stp[si[j]] = (uint16_t)(j * CT + tid);
  }
  __syncthreads();
  const uint32_t nt = (n - base) < (uint64_t)CU ? (uint32_t)(n - base) : (uint32_t)CU;
  for (uint32_t k = tid; k < nt; k += CT) {
    tmp[base + k] = stg[k];
    perm[base + k] = stp[k];
  }
}

// This batch's extent of cell c (a full warp calls it, c >= n_cells allowed: no cell): carved
// out of the bump arena (warp-aggregated), linked at the head of the cell's chain.
__device__ __forceinline__ void alloc_cell_warp(const DevGraph& g, const DevState& s, uint32_t c, bool err) {
  uint32_t cnt = (c < g.n_cells) ? s.bcount[c * BCOUNT_STRIDE] : 0;
  if (err) {
    if (c < g.n_cells && cnt) {
      s.bcount[c * BCOUNT_STRIDE] = 0;
      s.bcount[c * BCOUNT_STRIDE + 1] = 0;
    }
    return;
  }
  unsigned lane = threadIdx.x & 31;
  // extents start on 4-record boundaries so the flush can use 128-bit loads
  uint32_t alloc = (cnt + 3u) & ~3u;
  uint32_t incl = alloc;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= (unsigned)o) incl += y;
  }
  uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
  unsigned nonempty = __ballot_sync(0xffffffffu, cnt > 0);
  if (nonempty == 0) return;
  unsigned long long base = 0;
  unsigned ebase = 0;
  if (lane == 0) {
    base = atomicAdd(&s.st->arena_top, (unsigned long long)total);
    ebase = atomicAdd(&s.st->ext_top, (unsigned)__popc(nonempty));
  }
  base = __shfl_sync(0xffffffffu, base, 0);
  ebase = __shfl_sync(0xffffffffu, ebase, 0);
  if (cnt == 0) return;
  unsigned long long start = base + (incl - alloc);
  unsigned e = ebase + __popc(nonempty & lanemask_lt());
  if (start + alloc > s.ar.cap || e >= s.ext_cap) {  // host pre-checks make this unreachable
    atomicOr(&s.st->ingest_err, (unsigned)ERR_ARENA);
    return;
  }
  s.x_start[e] = (uint32_t)start;
  s.x_len[e] = cnt;
  s.x_tmax[e] = s.bcount[c * BCOUNT_STRIDE + 1];
  s.bcount[c * BCOUNT_STRIDE + 1] = 0;
  s.x_next[e] = s.cell_head[c];
  s.cell_head[c] = e;
  s.cell_pending[c] += cnt;
  s.bbase[c] = (uint32_t)start;
  s.bcount[c * BCOUNT_STRIDE] = 0;
}

// an accepted batch's newest t becomes t_now of the expiry rule (a rejected one changes nothing)
__device__ __forceinline__ void commit_batch_tmax(const DevState& s, bool err) {
  if (!err && blockIdx.x == 0 && threadIdx.x == 0) {
    const unsigned bt = *((volatile unsigned*)&s.st->batch_tmax);
    if (bt) atomicMax(&s.st->t_max, bt);
  }
}

__global__ void __launch_bounds__(256) k_ingest_alloc(DevGraph g, DevState s) {
  const bool err = s.st->ingest_err != 0;
  commit_batch_tmax(s, err);
  alloc_cell_warp(g, s, blockIdx.x * blockDim.x + threadIdx.x, err);
}

// One CTA per classify tile.  The tile's updates are staged in shared memory (coalesced), then
// thread k takes the k-th update in cell order: consecutive threads write consecutive
// positions of a cell's extent (coalesced runs, few pages per warp store).
__global__ void __launch_bounds__(CT) k_ingest_scatter(const uint4* __restrict__ upd, uint64_t n,
                                                       uint32_t seq0, DevGraph g, DevState s,
                                                       const uint2* __restrict__ tmp,
                                                       const uint16_t* __restrict__ perm) {
  extern __shared__ uint4 su[];  // CU records (SCATTER_SMEM bytes)
  const int tid = threadIdx.x;
  const uint64_t base = (uint64_t)blockIdx.x * CU;
  const uint32_t nt = (n - base) < (uint64_t)CU ? (uint32_t)(n - base) : (uint32_t)CU;
  // the tile's sorted (vertex, rank) and permutation (failed updates were left out: the
  // batch is rejected below then)
  uint2 vr[CPT];
  uint32_t il[CPT];
#pragma unroll
  for (int j = 0; j < CPT; ++j) {
    const uint32_t k = (uint32_t)(j * CT + tid);
    if (k < nt) {
      su[k] = __ldcs(upd + base + k);
      vr[j] = __ldcs(tmp + base + k);
      il[j] = __ldcs(perm + base + k);
    }
  }
  if (*((volatile unsigned*)&s.st->ingest_err)) return;
  __syncthreads();
  // two halves of CPT/2 updates: every load of a half in flight before its stores, at half
  // the registers (occupancy)
  constexpr int HP = CPT / 2;
#pragma unroll
  for (int hf = 0; hf < 2; ++hf) {
    uint32_t pos[HP];
    uint4 m[HP];
    unsigned long long cur[HP];
#pragma unroll
    for (int q = 0; q < HP; ++q) {
      const int j = hf * HP + q;
      const uint32_t k = (uint32_t)(j * CT + tid);
      if (k < nt) {
        m[q] = su[il[j]];
        pos[q] = vr[j].y == NONE ? NONE : s.bbase[cellof(g, vr[j].x)] + vr[j].y;
        cur[q] = __ldcg(s.ot_key + m[q].x);  // L2 value (the atomics' point of coherence)
      }
    }
#pragma unroll
    for (int q = 0; q < HP; ++q) {
      const int j = hf * HP + q;
      const uint32_t k = (uint32_t)(j * CT + tid);
      if (k >= nt) continue;
      const unsigned long long key =
          ((unsigned long long)m[q].w << 32) | (unsigned long long)(seq0 + (uint32_t)(base + il[j]));
      mark_moved(s, m[q].x, cellof(g, vr[j].x));
      if (pos[q] != NONE) {  // (NONE: a cell another rank owns)
        s.ar.obj[pos[q]] = m[q].x;
        s.ar.key[pos[q]] = key;
        s.ar.vsrc[pos[q]] = vr[j].x;
        s.ar.off[pos[q]] = m[q].z;
        s.ar.edge[pos[q]] = m[q].y;
      }
      // ot_key only grows: a key below the value already seen needs no atomic; a live object
      // takes a fire-and-forget RED.MAX; only an object seen without updates (0) needs the
      // old value back, to count it live exactly once
      if (cur[q] == 0ull) {
        const unsigned long long old = atomicMax(&s.ot_key[m[q].x], key);
        if (old == 0ull && key != 0ull) atomicAdd(&s.st->n_live, 1u);
      } else if (key > cur[q]) {
        atomicMax(&s.ot_key[m[q].x], key);
      }
    }
  }
}

static uint16_t* perm_of(uint2* tmp, uint64_t n) { return reinterpret_cast<uint16_t*>(tmp + n); }
size_t ingest_tmp_bytes(uint64_t n) { return (size_t)n * (sizeof(uint2) + sizeof(uint16_t)); }
void launch_ingest_classify(const uint4* upd, uint64_t n, const DevGraph& g, const DevState& s,
                            uint2* tmp, cudaStream_t st) {
  func_attr_once(k_ingest_classify, cudaFuncAttributeMaxDynamicSharedMemorySize, CLASSIFY_SMEM);
  unsigned blocks = (unsigned)((n + CU - 1) / CU);
  k_ingest_classify<<<blocks, CT, CLASSIFY_SMEM, st>>>(upd, n, g, s, tmp, perm_of(tmp, n));
}
void launch_ingest_alloc(const DevGraph& g, const DevState& s, cudaStream_t st) {
  k_ingest_alloc<<<(g.n_cells + 255) / 256, 256, 0, st>>>(g, s);
}
void launch_ingest_scatter(const uint4* upd, uint64_t n, uint32_t seq0, const DevGraph& g,
                           const DevState& s, const uint2* tmp, cudaStream_t st) {
  func_attr_once(k_ingest_scatter, cudaFuncAttributeMaxDynamicSharedMemorySize, SCATTER_SMEM);
  unsigned blocks = (unsigned)((n + CU - 1) / CU);
  k_ingest_scatter<<<blocks, CT, SCATTER_SMEM, st>>>(upd, n, seq0, g, s, tmp,
                                          perm_of(const_cast<uint2*>(tmp), n));
}

// ---------------------------------------------------------------------------------------
// Single-launch ingest for a batch that fits one resident wave: the classify, alloc and
// scatter phases above as one persistent cooperative kernel (one 1,024-thread CTA per SM)
// with two grid barriers between them.  Each CTA keeps its tile's cell hash, cell order and
// permutation in shared memory across the barriers (no tmp/perm round trip through HBM, no
// launch gaps, no tail wave); the scatter re-reads the tile's records from L2.
constexpr int FT = 1024;                // threads per CTA
constexpr int FPT = 8;                  // updates per thread at most
constexpr uint32_t FUSED_TILE = FT * FPT;
constexpr uint32_t FUSED_CH_MAX = 16384;  // cell-hash slots (>= 2 x distinct cells of a tile)

__device__ __forceinline__ void grid_barrier(unsigned* ctr, unsigned target) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(ctr, 1u);
    unsigned v;
    for (;;) {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
      if (v >= target) break;
      __nanosleep(64);
    }
  }
  __syncthreads();
}

__global__ void __launch_bounds__(FT, 1) k_ingest_fused(const uint4* __restrict__ upd, uint64_t n,
                                                        uint32_t seq0, uint32_t tile, uint32_t ch,
                                                        DevGraph g, DevState s) {
  extern __shared__ __align__(16) uint32_t f_buf[];
  uint32_t* h_cell = f_buf;          // [ch] cell id (REMOTE_CELL: other ranks' updates)
  uint32_t* h_cnt = f_buf + ch;      // [ch] count; after the scan (tile offset << 16) | count
  uint32_t* h_aux = f_buf + 2 * ch;  // [ch] newest t; then the cell's batch rank base; then the
                                     //      arena position of the group's first record minus its
                                     //      tile offset
  // (the tile's records are not staged: the scatter re-reads them from L2 -- the batch was just
  // read -- which leaves shared memory to a hash of >= one slot per update of the tile)
  uint2* stg = reinterpret_cast<uint2*>(f_buf + 3 * ch);    // [tile] (src vertex, slot | flags),
                                                            //        cell order
  uint16_t* stp = reinterpret_cast<uint16_t*>(stg + tile);  // [tile] tile index, cell order
  uint32_t* w_sum = reinterpret_cast<uint32_t*>(stp + ((tile + 1) & ~1u));  // [FT / 32]
  pdl_wait();   // (a programmatic dependent of the batch's status reset)
  pdl_allow();  // the next kernel (a knn round's status reset) may launch; it waits for this grid
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const unsigned G = gridDim.x;
  for (uint32_t i = tid; i < ch; i += FT) {
    h_cell[i] = NONE;
    h_cnt[i] = 0;
    h_aux[i] = 0;
  }
  __syncthreads();
  const uint64_t base = (uint64_t)blockIdx.x * tile;
  const uint32_t nt = base >= n ? 0u : (uint32_t)min((uint64_t)tile, n - base);

  // ---- classify: validate, cell via the inverted index, rank within the tile's cell group;
  //      the object's current key is read here too (in the same memory round as the inverted
  //      index): ot_key only grows, so "not newer than this value" still means no atomic is
  //      needed at the scatter, and a value of 0 marks a possibly new object
  uint32_t sr[FPT];  // (hash slot << 16) | rank in the slot's group, NONE: no record
  uint32_t vs[FPT];
  uint32_t fl = 0;   // 2 bits per update: 1 = newer than the key read, 2 = key read was 0
  uint32_t tl = 0;
  constexpr int HP = FPT / 2;
#pragma unroll
  for (int hf = 0; hf < 2; ++hf) {  // two halves: a half's loads and gathers in flight together
    uint4 mm[HP];
    uint2 ee[HP];
    unsigned long long ck[HP];
#pragma unroll
    for (int q = 0; q < HP; ++q) {
      const uint32_t k = (uint32_t)((hf * HP + q) * FT + tid);
      mm[q] = k < nt ? __ldg(upd + base + k) : make_uint4(0, 0xFFFFFFFFu, 0, 0);  // (kept in L2: re-read)
    }
#pragma unroll
    for (int q = 0; q < HP; ++q) {
      ee[q] = mm[q].y < g.A ? __ldg(g.einfo + mm[q].y) : make_uint2(0, 1);
      ck[q] = mm[q].x < s.max_objects ? __ldcg(s.ot_key + mm[q].x) : 0ull;
    }
#pragma unroll
    for (int q = 0; q < HP; ++q) {
      const int j = hf * HP + q;
      const uint32_t k = (uint32_t)(j * FT + tid);
      sr[j] = NONE;
      vs[j] = 0;
      if (k >= nt) continue;
      const uint4 m = mm[q];
      const uint2 e = ee[q];
      unsigned bad = 0;
      if (m.x >= s.max_objects) bad |= ERR_OBJ;
      if (m.y >= g.A) {
        bad |= ERR_EDGE;
      } else if (m.z >= e.y) {
        bad |= ERR_OFF;
      }
      if (bad) {
        const uint64_t i = base + k;
        atomicOr(&s.st->ingest_err, bad);
        atomicMin(&s.st->bad_index, i < 0xFFFFFFFFull ? (unsigned)i : 0xFFFFFFFFu);
        continue;
      }
      const unsigned long long key =
          ((unsigned long long)m.w << 32) | (unsigned long long)(seq0 + (uint32_t)(base + k));
      fl |= ((key > ck[q] ? 1u : 0u) | (ck[q] == 0ull ? 2u : 0u)) << (2 * j);
      const uint32_t c0 = cellof(g, e.x);
      const bool remote = s.n_ranks > 1 && owner_of(c0, g.n_cells, s.n_ranks) != s.rank;
      const uint32_t c = remote ? REMOTE_CELL : c0;
      uint32_t h = __umulhi(c * 2654435761u, ch);
      volatile uint32_t* vc = h_cell;
      for (;;) {
        const uint32_t cur = vc[h];
        if (cur == c) break;
        if (cur == NONE) {
          const uint32_t old = atomicCAS(&h_cell[h], NONE, c);
          if (old == NONE || old == c) break;
        }
        h = (h + 1) & (ch - 1);
      }
      sr[j] = (h << 16) | atomicAdd(&h_cnt[h], 1u);
      vs[j] = e.x;
      atomicMax(&h_aux[h], m.w);
      tl = max(tl, m.w);
    }
  }
  tl = __reduce_max_sync(0xffffffffu, tl);
  if (lane == 0 && tl) atomicMax(&s.st->batch_tmax, tl);  // (folded into t_max once accepted)
  __syncthreads();
  {  // exclusive scan of the slot counts = each group's offset in the tile's cell order
    const uint32_t spc = ch / FT;
    uint32_t sum = 0;
    for (uint32_t q = 0; q < spc; ++q) sum += h_cnt[tid * spc + q];
    uint32_t x = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) w_sum[wid] = x;
    __syncthreads();
    uint32_t run = x - sum;
    for (int w = 0; w < wid; ++w) run += w_sum[w];
    for (uint32_t q = 0; q < spc; ++q) {
      const uint32_t c = h_cnt[tid * spc + q];
      h_cnt[tid * spc + q] = c | (run << 16);  // (counts and offsets <= FUSED_TILE < 2^16)
      run += c;
    }
  }
  __syncthreads();  // (the claims below read other threads' slots)
  // one claim per distinct cell of the tile on the batch counters
  for (uint32_t i = tid; i < ch; i += FT) {
    const uint32_t c = h_cell[i];
    if (c != NONE && c != REMOTE_CELL) {
      atomicMax(&s.bcount[c * BCOUNT_STRIDE + 1], h_aux[i]);
      h_aux[i] = atomicAdd(&s.bcount[c * BCOUNT_STRIDE], h_cnt[i] & 0xFFFFu);
    }
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < FPT; ++j) {
    if (sr[j] == NONE) continue;
    const uint32_t slot = sr[j] >> 16;
    const uint32_t si = (h_cnt[slot] >> 16) + (sr[j] & 0xFFFFu);
    stg[si] = make_uint2(vs[j], slot | (((fl >> (2 * j)) & 3u) << 16));
    stp[si] = (uint16_t)(j * FT + tid);
  }

  // ---- alloc: every tile's counts are in; one extent per (batch, cell)
  grid_barrier(&s.st->ingest_bar, G);
  {
    const bool err = *((volatile unsigned*)&s.st->ingest_err) != 0;
    commit_batch_tmax(s, err);
    const uint32_t nw = G * (FT / 32);
    for (uint32_t c0 = (blockIdx.x * (FT / 32) + wid) * 32; c0 < g.n_cells; c0 += nw * 32)
      alloc_cell_warp(g, s, c0 + lane, err);
  }
  grid_barrier(&s.st->ingest_bar, 2 * G);
  if (*((volatile unsigned*)&s.st->ingest_err)) return;  // the batch is rejected as a whole

  // ---- scatter in cell order (consecutive threads write consecutive extent positions);
  //      everything it reads is in shared memory but the extents' bases (one per group)
  for (uint32_t i = tid; i < ch; i += FT) {
    const uint32_t c = h_cell[i];
    if (c != NONE && c != REMOTE_CELL) h_aux[i] = s.bbase[c] + h_aux[i] - (h_cnt[i] >> 16);
  }
  __syncthreads();
#pragma unroll 4
  for (uint32_t si = tid; si < nt; si += FT) {
    const uint2 x = stg[si];
    const uint32_t k = stp[si];
    const uint4 m = __ldg(upd + base + k);
    const uint32_t slot = x.y & 0xFFFFu, f = x.y >> 16;
    const unsigned long long key =
        ((unsigned long long)m.w << 32) | (unsigned long long)(seq0 + (uint32_t)(base + k));
    mark_moved(s, m.x, cellof(g, x.x));
    if (h_cell[slot] != REMOTE_CELL) {  // (REMOTE_CELL: a cell another rank owns)
      const uint32_t pos = h_aux[slot] + si;
      s.ar.obj[pos] = m.x;
      s.ar.key[pos] = key;
      s.ar.vsrc[pos] = x.x;
      s.ar.off[pos] = m.z;
      s.ar.edge[pos] = m.y;
    }
    // ot_key only grows: a key not above the value read needs no atomic; a live object takes a
    // fire-and-forget RED.MAX; only an object read as 0 needs the old value back, to count it
    // live exactly once
    if (f & 2u) {
      const unsigned long long old = atomicMax(&s.ot_key[m.x], key);
      if (old == 0ull && key != 0ull) atomicAdd(&s.st->n_live, 1u);
    } else if (f & 1u) {
      atomicMax(&s.ot_key[m.x], key);
    }
  }
}

// ---------------------------------------------------------------------------------------
// Direct single-launch ingest for a batch of at most one resident wave x DPT updates whose
// tiles hit nearly as many distinct cells as they hold updates (C3's step: 1M updates over
// 23k cells, ~0.3 updates per (tile, cell)), where a per-tile cell hash aggregates nothing and
// only adds its shared-memory passes: every update takes its rank in its cell's batch extent
// with one returning atomic on the cell's counter line, keeps (cell, rank, source vertex) in
// registers across the two grid barriers (no shared memory, no tmp/perm round trip), and the
// scatter re-reads its record from L2.  Same arithmetic and rejection rules as the paths above.
constexpr int DT = 512;   // threads per CTA (2 CTAs per SM)
#ifndef GG_DIRECT_HP
#define GG_DIRECT_HP 2
#endif
// (experiment hook) GG_INGEST_TIMING=1: phase timestamps of the first and last CTA, printed
#ifndef GG_INGEST_TIMING
#define GG_INGEST_TIMING 0
#endif
#if GG_INGEST_TIMING
#define DTIME(k) unsigned long long _t##k; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(_t##k))
#define DTIME_PRINT()                                                                              \
  if (threadIdx.x == 0 && (blockIdx.x == 0 || blockIdx.x == gridDim.x - 1))                        \
    printf("ingest_direct cta %u: p1 %llu bar1 %llu alloc %llu bar2 %llu scatter %llu ns\n", blockIdx.x, \
           _t1 - _t0, _t2 - _t1, _t3 - _t2, _t4 - _t3, _t5 - _t4)
#else
#define DTIME(k)
#define DTIME_PRINT()
#endif
constexpr int DPT = 8;    // updates per thread at most
// rank flags: a cell another rank owns / key newer than the one read / key read was 0
constexpr uint32_t RK_REMOTE = 1u << 29, RK_NEW = 1u << 30, RK_ZERO = 1u << 31;
constexpr uint32_t RK_MASK = RK_REMOTE - 1;

__global__ void __launch_bounds__(DT, 2) k_ingest_direct(const uint4* __restrict__ upd, uint64_t n,
                                                         uint32_t seq0, DevGraph g, DevState s) {
  pdl_wait();   // (a programmatic dependent of the batch's status reset)
  pdl_allow();  // the next kernel may launch; it waits for this grid
  DTIME(0);
  const uint32_t T = gridDim.x * DT;
  const uint32_t tid = blockIdx.x * DT + threadIdx.x;
  const int lane = threadIdx.x & 31;
  // per update: source vertex (NONE: no update; its cell is cellof), rank | flags, and the cell
  // whose cleaned list the object leaves (R8's STALE mark; NONE: none)
  uint32_t rk[DPT], vs[DPT], lv[DPT];
  uint32_t tl = 0;
  constexpr int HP = GG_DIRECT_HP;  // (parts: registers vs gathers in flight)
#pragma unroll
  for (int hf = 0; hf < DPT / HP; ++hf) {  // a part's loads and gathers in flight together
    uint4 mm[HP];
    uint2 ee[HP];
    unsigned long long ck[HP];
    uint32_t lc[HP];
#pragma unroll
    for (int q = 0; q < HP; ++q) {
      const uint64_t i = (uint64_t)(hf * HP + q) * T + tid;
      mm[q] = i < n ? __ldg(upd + i) : make_uint4(0, 0xFFFFFFFFu, 0, 0);  // (re-read from L2)
    }
#pragma unroll
    for (int q = 0; q < HP; ++q) {  // one memory round: inverted index, object key, listed cell
      const bool ok = mm[q].x < s.max_objects;
      ee[q] = mm[q].y < g.A ? __ldg(g.einfo + mm[q].y) : make_uint2(0, 1);
      ck[q] = ok ? __ldcg(s.ot_key + mm[q].x) : 0ull;
      lc[q] = ok ? s.listed_cell[mm[q].x] : NONE;
    }
#pragma unroll
    for (int q = 0; q < HP; ++q) {
      const int j = hf * HP + q;
      const uint64_t i = (uint64_t)j * T + tid;
      rk[j] = 0;
      vs[j] = NONE;
      lv[j] = NONE;
      if (i >= n) continue;
      const uint4 m = mm[q];
      const uint2 e = ee[q];
      unsigned bad = 0;
      if (m.x >= s.max_objects) bad |= ERR_OBJ;
      if (m.y >= g.A) {
        bad |= ERR_EDGE;
      } else if (m.z >= e.y) {
        bad |= ERR_OFF;
      }
      if (bad) {
        atomicOr(&s.st->ingest_err, bad);
        atomicMin(&s.st->bad_index, i < 0xFFFFFFFFull ? (unsigned)i : 0xFFFFFFFFu);
        continue;
      }
      const unsigned long long key = ((unsigned long long)m.w << 32) | (unsigned long long)(seq0 + (uint32_t)i);
      const uint32_t c0 = cellof(g, e.x);
      const bool remote = s.n_ranks > 1 && owner_of(c0, g.n_cells, s.n_ranks) != s.rank;
      vs[j] = e.x;
      lv[j] = (lc[q] != NONE && lc[q] != c0) ? lc[q] : NONE;
      rk[j] = (key > ck[q] ? RK_NEW : 0u) | (ck[q] == 0ull ? RK_ZERO : 0u) | (remote ? RK_REMOTE : 0u);
      if (!remote) atomicMax(&s.bcount[c0 * BCOUNT_STRIDE + 1], m.w);  // the extent's zeta.t
      tl = max(tl, m.w);
    }
  }
  // ranks: one returning atomic per update, all of a thread's in flight together
#pragma unroll
  for (int j = 0; j < DPT; ++j) {
    if (vs[j] != NONE && !(rk[j] & RK_REMOTE)) rk[j] |= atomicAdd(&s.bcount[cellof(g, vs[j]) * BCOUNT_STRIDE], 1u);
  }
  tl = __reduce_max_sync(0xffffffffu, tl);
  if (lane == 0 && tl) atomicMax(&s.st->batch_tmax, tl);  // (folded into t_max once accepted)

  // ---- alloc: every rank is taken; one extent per (batch, cell)
  const unsigned G = gridDim.x;
  DTIME(1);
  grid_barrier(&s.st->ingest_bar, G);
  DTIME(2);
  {
    const bool err = *((volatile unsigned*)&s.st->ingest_err) != 0;
    commit_batch_tmax(s, err);
    // an accepted batch marks the cells its objects leave STALE (mark_moved; a cell that also gets
    // an extent here is dirty either way, so the order against the allocation does not matter)
    if (!err) {
#pragma unroll
      for (int j = 0; j < DPT; ++j)
        if (lv[j] != NONE) atomicCAS(&s.cell_head[lv[j]], NONE, STALE);
    }
    const uint32_t nw = G * (DT / 32);
    for (uint32_t c0 = (blockIdx.x * (DT / 32) + (threadIdx.x >> 5)) * 32; c0 < g.n_cells; c0 += nw * 32)
      alloc_cell_warp(g, s, c0 + lane, err);
  }
  DTIME(3);
  grid_barrier(&s.st->ingest_bar, 2 * G);
  DTIME(4);
  if (*((volatile unsigned*)&s.st->ingest_err)) return;  // the batch is rejected as a whole

  // ---- scatter: record j of this thread to its cell's extent at bbase + rank (parts of 4: every
  //      load of a part in flight before its stores)
  uint32_t* __restrict__ a_obj = s.ar.obj;
  unsigned long long* __restrict__ a_key = s.ar.key;
  uint32_t* __restrict__ a_vsrc = s.ar.vsrc;
  uint32_t* __restrict__ a_off = s.ar.off;
  uint32_t* __restrict__ a_edge = s.ar.edge;
  constexpr int SP = 4;
#pragma unroll
  for (int h = 0; h < DPT / SP; ++h) {
    uint4 m[SP];
    uint32_t pos[SP];
#pragma unroll
    for (int q = 0; q < SP; ++q) {
      const int j = h * SP + q;
      const uint64_t i = (uint64_t)j * T + tid;
      const bool own = vs[j] != NONE && !(rk[j] & RK_REMOTE);
      m[q] = vs[j] != NONE ? __ldg(upd + i) : make_uint4(0, 0, 0, 0);
      pos[q] = own ? __ldcg(s.bbase + cellof(g, vs[j])) + (rk[j] & RK_MASK) : NONE;
    }
#pragma unroll
    for (int q = 0; q < SP; ++q) {
      const int j = h * SP + q;
      if (vs[j] == NONE) continue;
      const uint64_t i = (uint64_t)j * T + tid;
      const unsigned long long key = ((unsigned long long)m[q].w << 32) | (unsigned long long)(seq0 + (uint32_t)i);
      if (pos[q] != NONE) {  // (NONE: a cell another rank owns)
        a_obj[pos[q]] = m[q].x;
        a_key[pos[q]] = key;
        a_vsrc[pos[q]] = vs[j];
        a_off[pos[q]] = m[q].z;
        a_edge[pos[q]] = m[q].y;
      }
      if (rk[j] & RK_ZERO) {
        const unsigned long long old = atomicMax(&s.ot_key[m[q].x], key);
        if (old == 0ull && key != 0ull) atomicAdd(&s.st->n_live, 1u);
      } else if (rk[j] & RK_NEW) {
        atomicMax(&s.ot_key[m[q].x], key);
      }
    }
  }
  DTIME(5);
  DTIME_PRINT();
}

// a tile whose 2-slots-per-cell hash does not fit shared memory: fused with a hash of one slot
// per update (1) or the three-launch path (0; measured faster at C3's 1M-update step, r2i: 0.144
// vs 0.170 ms -- probe chains at 82% load)
#ifndef GG_FUSED_TIGHT
#define GG_FUSED_TIGHT 0
#endif
static size_t fused_smem(uint32_t tile, uint32_t ch) {
  return (size_t)ch * 12 + (size_t)tile * 8 + (size_t)((tile + 1) & ~1u) * 2 + (FT / 32) * 4;
}

// mode: 0 = choose (direct when an SM tile would average under two updates per distinct cell),
// 1 = the cell-hash launch only, 2 = the direct launch whenever it fits
bool ingest_fused_plan(uint64_t n, uint32_t n_cells, int sm_count, int mode, IngestPlan* p) {
  if (n == 0 || sm_count <= 0) return false;
  p->direct = false;
  const uint64_t dgrid = (uint64_t)sm_count * 2;  // (2 CTAs of DT threads per SM)
  if (mode != 1 && n <= dgrid * DT * DPT) {
    const uint64_t tile = (n + sm_count - 1) / sm_count;  // a cell-hash tile: one CTA per SM
    if (mode == 2 || tile <= 2ull * n_cells) {
      p->direct = true;
      // >= 2 updates per thread (all SMs once the batch is large); dgrid x DT x DPT >= n
      p->grid = (uint32_t)std::min<uint64_t>(dgrid, (n + 2ull * DT - 1) / (2ull * DT));
      p->tile = 0;
      p->ch = 0;
      p->smem = 0;
      return true;
    }
  }
  const uint64_t grid = std::min<uint64_t>((uint64_t)sm_count, std::max<uint64_t>(1, (n + 2047) / 2048));
  const uint64_t tile = (n + grid - 1) / grid;
  if (tile > FUSED_TILE) return false;
  // cell-hash slots: >= 2 per distinct cell of a tile when that fits, else >= one more than the
  // tile's updates (never full: at most one distinct cell per update; C3's 1M-update step, 6,757
  // updates per tile over 23k cells, takes 8,192 slots)
  const uint64_t m = std::min<uint64_t>(tile, (uint64_t)n_cells + 1);
  uint32_t ch = FT;
  while (ch < 2 * m) ch <<= 1;
  if (GG_FUSED_TIGHT && (ch > FUSED_CH_MAX || fused_smem((uint32_t)tile, ch) > 227 * 1024)) {
    ch = FT;
    while (ch < m + 1) ch <<= 1;
  }
  if (ch > FUSED_CH_MAX) return false;
  const size_t smem = fused_smem((uint32_t)tile, ch);
  if (smem > 227 * 1024) return false;
  p->grid = (uint32_t)grid;
  p->tile = (uint32_t)tile;
  p->ch = ch;
  p->smem = smem;
  return true;
}

cudaError_t launch_ingest_fused(const uint4* upd, uint64_t n, uint32_t seq0, const DevGraph& g,
                                const DevState& s, const IngestPlan& p, cudaStream_t st) {
  if (p.direct) {
    cudaLaunchAttribute attr[2];
    cudaLaunchConfig_t cfg = pdl_config(dim3(p.grid), dim3(DT), 0, st, attr);
    attr[1].id = cudaLaunchAttributeCooperative;
    attr[1].val.cooperative = 1;
    cfg.numAttrs = 2;
    return cudaLaunchKernelEx(&cfg, k_ingest_direct, upd, n, seq0, g, s);
  }
  const cudaError_t ae = func_attr_once(k_ingest_fused, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
  if (ae != cudaSuccess) return ae;
  // cooperative (every CTA resident at once, or the launch fails: the grid barriers need it) and
  // a programmatic dependent of the batch's status reset
  cudaLaunchAttribute attr[2];
  cudaLaunchConfig_t cfg = pdl_config(dim3(p.grid), dim3(FT), p.smem, st, attr);
  attr[1].id = cudaLaunchAttributeCooperative;
  attr[1].val.cooperative = 1;
  cfg.numAttrs = 2;
  return cudaLaunchKernelEx(&cfg, k_ingest_fused, upd, n, seq0, p.tile, p.ch, g, s);
}

// ---------------------------------------------------------------------------------------
// Alg. 4 line 1 (P@45660): c_q = getCell(q.e) and getNeighbors({c_q}) are cleaned first.
// mode SEED_NEIGHBORS: c_q and its neighbour cells per query; SEED_DST: c_q and the cell of the
// query arc's head; SEED_ALL: every dirty cell, each requested once by thread c (a batch large
// enough to touch nearly every cell: one uncontended request per cell instead of ~n_q x 9
// racing on the same cells).  Every mode validates the queries and copies mapped ones.
__global__ void __launch_bounds__(256) k_seed(const uint2* __restrict__ q, uint32_t nq, DevGraph g,
                                              DevState s, uint32_t epoch, int mode,
                                              uint2* __restrict__ q_copy) {
  pdl_wait();   // (launched as a programmatic dependent of the round's status reset)
  pdl_allow();  // the flush may launch now (it waits for this grid before reading)
  uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (mode == SEED_ALL && i < g.n_cells) request_flush(s, i, epoch);
  if (i >= nq) return;
  uint2 qq = q[i];
  // queries in mapped host memory are read across PCIe once, here, and kept in HBM for the
  // expansion (each warp re-reading its query over PCIe would queue behind a staged transfer)
  if (q_copy) q_copy[i] = qq;
  if (qq.x >= g.A) {
    atomicOr(&s.st->err, (unsigned)ERR_QUERY);
    return;
  }
  uint2 e = g.einfo[qq.x];
  if (qq.y >= e.y) {
    atomicOr(&s.st->err, (unsigned)ERR_QUERY);
    return;
  }
  if (mode == SEED_ALL) return;
  uint32_t c = cellof(g, e.x);
  request_flush(s, c, epoch);
  if (mode == SEED_NEIGHBORS) {
    for (uint32_t j = g.cadj_ptr[c]; j < g.cadj_ptr[c + 1]; ++j) request_flush(s, g.cadj[j], epoch);
  } else {
    request_flush(s, cellof(g, g.edst[qq.x]), epoch);
  }
}

void launch_seed(const uint2* q, uint32_t nq, const DevGraph& g, const DevState& s, uint32_t epoch,
                 int mode, uint2* q_copy, cudaStream_t st) {
  const uint32_t n = mode == SEED_ALL ? std::max(nq, g.n_cells) : nq;
  if (n == 0) return;
  cudaLaunchAttribute attr[1];
  const cudaLaunchConfig_t cfg = pdl_config(dim3((n + 255) / 256), dim3(256), 0, st, attr);
  cudaLaunchKernelEx(&cfg, k_seed, q, nq, g, s, epoch, mode, q_copy);
}

// Arrival-index re-base (api.cu rebase(): right after a garbage collection)
__global__ void __launch_bounds__(256) k_rebase_keys(DevState s, unsigned long long n_records) {
  const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
  for (unsigned long long i = blockIdx.x * blockDim.x + threadIdx.x; i < n_records + s.max_objects; i += stride) {
    unsigned long long* p = i < n_records ? s.ar.key + i : s.ot_key + (i - n_records);
    const unsigned long long k = *p;
    if (k) *p = (k & 0xFFFFFFFF00000000ull) | 1ull;
  }
}
void launch_rebase_keys(const DevState& s, unsigned long long n_records, cudaStream_t st) {
  k_rebase_keys<<<148 * 8, 256, 0, st>>>(s, n_records);
}

// Every dirty cell (eager cleaning; all_cells additionally queues clean cells for GC).
__global__ void __launch_bounds__(256) k_mark_dirty(DevGraph g, DevState s, uint32_t epoch,
                                                    int all_cells) {
  uint32_t c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= g.n_cells) return;
  bool want = all_cells ? true : (s.cell_head[c] != NONE);
  if (!want) return;
  unsigned act = __activemask();
  int leader = __ffs(act) - 1;
  unsigned base = 0;
  if ((int)(threadIdx.x & 31) == leader) base = atomicAdd(&s.st->n_flush, (unsigned)__popc(act));
  base = __shfl_sync(act, base, leader);
  s.flush_list[base + __popc(act & lanemask_lt())] = c;
  s.cell_req[c] = epoch;
}

void launch_mark_dirty(const DevGraph& g, const DevState& s, uint32_t epoch, int all_cells,
                       cudaStream_t st) {
  k_mark_dirty<<<(g.n_cells + 255) / 256, 256, 0, st>>>(g, s, epoch, all_cells);
}

// Valid objects of one clean cell (test hook ggrid_cell_objects).
__global__ void k_dump_cell(DevGraph g, DevState s, uint32_t c, uint32_t* obj, uint32_t* edge,
                            uint32_t* off, uint32_t cap, uint32_t* n_out) {
  uint32_t vb = c * g.cs;
  uint32_t ve = min(g.V, vb + g.cs);
  for (uint32_t v = vb + threadIdx.x; v < ve; v += blockDim.x) {
    uint2 vo = vobj_valid(s.v_obj[v], s.cell_comp[c]);
    for (uint32_t j = 0; j < vo.y; ++j) {
      uint32_t p = vo.x + j;
      uint32_t o = s.ar.obj[p];
      if (s.ar.key[p] != s.ot_key[o]) continue;  // moved away since the cell was cleaned
      uint32_t i = atomicAdd(n_out, 1u);
      if (i < cap) {
        obj[i] = o;
        edge[i] = s.ar.edge[p];
        off[i] = s.ar.off[p];
      }
    }
  }
}

void launch_dump_cell(const DevGraph& g, const DevState& s, uint32_t c, uint32_t* obj,
                      uint32_t* edge, uint32_t* off, uint32_t cap, uint32_t* n_out, cudaStream_t st) {
  k_dump_cell<<<1, 256, 0, st>>>(g, s, c, obj, edge, off, cap, n_out);
}

}  // namespace gg

namespace gg {
__global__ void k_set_words(WordSet ws) {
  pdl_wait();   // (a programmatic dependent of the ingest before a knn round)
  pdl_allow();  // a programmatic dependent (the seed / flush / ingest) may launch now
  if (ws.fold_dst && threadIdx.x == 0) *ws.fold_dst |= *ws.fold_src;
  __syncwarp();
  if ((int)threadIdx.x < ws.n) *ws.p[threadIdx.x] = ws.v[threadIdx.x];
}
void launch_set_words(const WordSet& ws, cudaStream_t st) {
  if (!ws.n && !ws.fold_dst) return;
  cudaLaunchAttribute attr[1];
  const cudaLaunchConfig_t cfg = pdl_config(dim3(1), dim3(32), 0, st, attr);
  cudaLaunchKernelEx(&cfg, k_set_words, ws);
}
}  // namespace gg

namespace gg {
// status readback through mapped pinned memory: a kernel store, no copy engine involved
__global__ void k_copy_words(const uint32_t* __restrict__ src, uint32_t* __restrict__ dst, int n) {
  for (int i = threadIdx.x; i < n; i += blockDim.x) dst[i] = src[i];
}
void launch_copy_words(const void* src, void* dst, size_t bytes, cudaStream_t st) {
  k_copy_words<<<1, 64, 0, st>>>(static_cast<const uint32_t*>(src), static_cast<uint32_t*>(dst),
                                 (int)(bytes / 4));
}
}  // namespace gg

namespace gg {
// owner rank of each query (cell of its arc's source vertex; sharded mode routing)
__global__ void k_query_owner(const uint2* __restrict__ q, uint32_t nq, DevGraph g, DevState s,
                              uint32_t* __restrict__ out) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nq) return;
  const uint32_t e = q[i].x;
  out[i] = e < g.A ? owner_of(cellof(g, g.einfo[e].x), g.n_cells, s.n_ranks) : 0u;
}
void launch_query_owner(const uint2* q, uint32_t nq, const DevGraph& g, const DevState& s,
                        uint32_t* out_rank, cudaStream_t st) {
  if (nq) k_query_owner<<<(nq + 255) / 256, 256, 0, st>>>(q, nq, g, s, out_rank);
}

// One warp per query: lane l < n_lists holds the head of list l; k rounds of a warp arg-min on
// (dist, obj) (the final first-k of the candidate union, P@49436-49765 / P@51679).
__global__ void k_merge_topk(uint32_t n_lists, uint32_t n_q, uint32_t k,
                             const uint32_t* __restrict__ lobj, const uint32_t* __restrict__ ldist,
                             uint32_t* __restrict__ out_obj, uint32_t* __restrict__ out_dist) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t qi = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (qi >= n_q) return;
  const size_t row = (size_t)qi * k;
  const size_t stride = (size_t)n_q * k;
  uint32_t head = 0;
  auto key_at = [&](uint32_t h) -> unsigned long long {
    if (lane >= n_lists || h >= k) return EMPTY64;
    const size_t p = lane * stride + row + h;
    return ((unsigned long long)ldist[p] << 32) | lobj[p];
  };
  unsigned long long cur = key_at(head);
  for (uint32_t r = 0; r < k; ++r) {
    const uint32_t dmin = __reduce_min_sync(0xffffffffu, (uint32_t)(cur >> 32));
    const uint32_t omin = __reduce_min_sync(0xffffffffu, (uint32_t)(cur >> 32) == dmin ? (uint32_t)cur : 0xFFFFFFFFu);
    const unsigned long long best = ((unsigned long long)dmin << 32) | omin;
    if (lane == 0) {
      out_obj[row + r] = best == EMPTY64 ? GGRID_PAD : omin;
      out_dist[row + r] = best == EMPTY64 ? GGRID_PAD : dmin;
    }
    if (best != EMPTY64 && cur == best) cur = key_at(++head);  // (lists are disjoint)
  }
}
void launch_merge_topk(uint32_t n_lists, uint32_t n_q, uint32_t k, const uint32_t* lobj,
                       const uint32_t* ldist, uint32_t* out_obj, uint32_t* out_dist, cudaStream_t st) {
  if (n_q) k_merge_topk<<<(n_q + 7) / 8, 256, 0, st>>>(n_lists, n_q, k, lobj, ldist, out_obj, out_dist);
}
}  // namespace gg

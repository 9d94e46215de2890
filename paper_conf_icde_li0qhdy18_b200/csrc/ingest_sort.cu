// ingest_sort.cu — caching a large update batch (Alg. 1, P@18177-19248) through a sort by cell.
//
// The three-launch path (ingest.cu) aggregates updates per cell inside 8,192-update tiles.  When a
// tile meets about as many distinct cells as it holds updates (C3: 23k cells, ~0.35 updates per
// (tile, cell)) that aggregation buys nothing: every tile still claims ~one counter per update and
// scatters its records one by one into ~23k extents (partial-sector writes, ~1.8x the algorithmic
// bytes).  Here the batch is ordered by cell first, so each cell's records of the batch are
// consecutive and every write is a coalesced run:
//   keys    : validate, cell(src(e)) via the inverted index (P@15006); key = cell, value =
//             (source vertex << 32 | batch index); the batch's newest t
//   sort    : radix sort of the (cell, value) pairs on the cell bits (CUB, the toolkit's primitive)
//   runs    : per cell of the sorted batch its record count and first sorted position (one atomic
//             per warp segment, not per update)
//   alloc   : k_ingest_alloc (ingest.cu), unchanged: one extent per (batch, cell)
//   scatter : sorted position i of cell c goes to bbase[c] + (i - first[c]); the new extent's
//             newest t by one atomicMax per warp segment; the object table takes the key by
//             RED.MAX (only when newer than the value read), STALE marks (reading R8)
// Same arithmetic, validation and whole-batch rejection as the other paths.
#include <cub/cub.cuh>

#include "internal.cuh"

namespace gg {

namespace {

constexpr int ST = 256;             // threads per CTA
constexpr uint32_t BC_FIRST = 2;    // bcount word: the cell's first position in the sorted batch

#ifndef GG_KPT
#define GG_KPT 8
#endif
constexpr int KPT = GG_KPT;  // updates per thread in the keys pass (their gathers in flight together)

__global__ void __launch_bounds__(ST) k_bulk_keys(const uint4* __restrict__ upd, uint64_t n, DevGraph g,
                                                  DevState s, uint32_t* __restrict__ keys,
                                                  unsigned long long* __restrict__ vals) {
  const uint64_t i0 = (uint64_t)blockIdx.x * (ST * KPT) + threadIdx.x;
  uint32_t tl = 0;
  uint4 mm[KPT];
  uint2 ee[KPT];
#pragma unroll
  for (int q = 0; q < KPT; ++q) {
    const uint64_t i = i0 + (uint64_t)q * ST;
    mm[q] = i < n ? __ldg(upd + i) : make_uint4(0, 0xFFFFFFFFu, 0, 0);
  }
#pragma unroll
  for (int q = 0; q < KPT; ++q) ee[q] = mm[q].y < g.A ? __ldg(g.einfo + mm[q].y) : make_uint2(0, 1);
#pragma unroll
  for (int q = 0; q < KPT; ++q) {
    const uint64_t i = i0 + (uint64_t)q * ST;
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
    uint32_t key = g.n_cells + 1;  // (invalid: sorted last, never scattered)
    if (bad) {
      atomicOr(&s.st->ingest_err, bad);
      atomicMin(&s.st->bad_index, i < 0xFFFFFFFFull ? (unsigned)i : 0xFFFFFFFFu);
    } else {
      const uint32_t c = cellof(g, e.x);
      // a cell another rank owns: sorted just past the real cells (object table update only)
      key = (s.n_ranks > 1 && owner_of(c, g.n_cells, s.n_ranks) != s.rank) ? g.n_cells : c;
      tl = max(tl, m.w);
    }
    keys[i] = key;
    vals[i] = ((unsigned long long)e.x << 32) | (uint32_t)i;  // (source vertex, batch index)
  }
  tl = __reduce_max_sync(0xffffffffu, tl);
  if ((threadIdx.x & 31) == 0 && tl) atomicMax(&s.st->batch_tmax, tl);  // (t_max once accepted)
}

// per warp segment of equal keys (the batch is sorted, so a segment is a run of lanes): one
// atomicAdd of its length on the cell's counter; the run's first element records its position
__global__ void __launch_bounds__(ST) k_bulk_runs(const uint32_t* __restrict__ keys, uint64_t n, DevGraph g,
                                                  DevState s) {
  if (*((volatile unsigned*)&s.st->ingest_err)) return;  // (rejected: alloc resets nothing of ours)
  const uint64_t i = (uint64_t)blockIdx.x * ST + threadIdx.x;
  const int lane = threadIdx.x & 31;
  const uint32_t c = i < n ? keys[i] : 0xFFFFFFFFu;
  const unsigned grp = __match_any_sync(0xffffffffu, c);
  if (c < g.n_cells) {
    if (lane == 31 - __clz(grp)) atomicAdd(&s.bcount[c * BCOUNT_STRIDE], (unsigned)__popc(grp));
    if (i == 0 || keys[i - 1] != c) s.bcount[c * BCOUNT_STRIDE + BC_FIRST] = (uint32_t)i;
  }
}

constexpr int SPT = 4;  // sorted records per thread in the scatter (gathers in flight together)

__global__ void __launch_bounds__(ST) k_bulk_scatter(const uint4* __restrict__ upd,
                                                     const uint32_t* __restrict__ keys,
                                                     const unsigned long long* __restrict__ vals, uint64_t n,
                                                     uint32_t seq0, DevGraph g, DevState s) {
  if (*((volatile unsigned*)&s.st->ingest_err)) return;  // the batch is rejected as a whole
  const uint64_t i0 = (uint64_t)blockIdx.x * (ST * SPT) + threadIdx.x;
  uint32_t cc[SPT], idx[SPT], vsrc[SPT];
  uint4 m[SPT];
#pragma unroll
  for (int q = 0; q < SPT; ++q) {
    const uint64_t i = i0 + (uint64_t)q * ST;
    cc[q] = i < n ? keys[i] : 0xFFFFFFFFu;
    const unsigned long long v = i < n ? vals[i] : 0ull;
    idx[q] = (uint32_t)v;
    vsrc[q] = (uint32_t)(v >> 32);
  }
#pragma unroll
  for (int q = 0; q < SPT; ++q) m[q] = cc[q] <= g.n_cells ? __ldg(upd + idx[q]) : make_uint4(0, 0, 0, 0);
  uint32_t first[SPT];
  unsigned long long cur[SPT];
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int q = 0; q < SPT; ++q) {
    const bool rec = cc[q] <= g.n_cells;  // (n_cells: a cell another rank owns; above: invalid)
    cur[q] = rec ? __ldcg(s.ot_key + m[q].x) : 0ull;
    first[q] = cc[q] < g.n_cells ? s.bcount[cc[q] * BCOUNT_STRIDE + BC_FIRST] : 0u;
    // the new extent's newest t (zeta.t of the expiry rule): one atomicMax per warp segment of
    // the sorted batch (the 32 records of this q are consecutive, a segment a run of lanes)
    uint32_t t = rec ? m[q].w : 0u;
    const unsigned grp = __match_any_sync(0xffffffffu, cc[q]);
    const int head = __ffs(grp) - 1;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t u = __shfl_up_sync(0xffffffffu, t, o);
      if (lane - o >= head) t = max(t, u);
    }
    if (cc[q] < g.n_cells && lane == 31 - __clz(grp)) atomicMax(&s.x_tmax[s.cell_head[cc[q]]], t);
  }
#pragma unroll
  for (int q = 0; q < SPT; ++q) {
    const uint32_t c = cc[q];
    if (c > g.n_cells) continue;
    const uint64_t i = i0 + (uint64_t)q * ST;
    const unsigned long long key = ((unsigned long long)m[q].w << 32) | (unsigned long long)(seq0 + idx[q]);
    mark_moved(s, m[q].x, cellof(g, vsrc[q]));
    if (c < g.n_cells) {
      const uint32_t pos = s.bbase[c] + ((uint32_t)i - first[q]);
      s.ar.obj[pos] = m[q].x;
      s.ar.key[pos] = key;
      s.ar.vsrc[pos] = vsrc[q];
      s.ar.off[pos] = m[q].z;
      s.ar.edge[pos] = m[q].y;
    }
    // ot_key only grows: no atomic for a key not above the value read; an object read as 0 takes
    // the returning form, to count it live exactly once
    if (cur[q] == 0ull) {
      const unsigned long long old = atomicMax(&s.ot_key[m[q].x], key);
      if (old == 0ull && key != 0ull) atomicAdd(&s.st->n_live, 1u);
    } else if (key > cur[q]) {
      atomicMax(&s.ot_key[m[q].x], key);
    }
  }
}

struct SortLayout {
  size_t keys, keys2, vals, vals2, temp, temp_bytes, total;
};
size_t align256(size_t x) { return (x + 255) & ~size_t(255); }
SortLayout sort_layout(uint64_t n, uint32_t n_cells) {
  SortLayout L;
  L.keys = 0;
  L.keys2 = align256(L.keys + n * 4);
  L.vals = align256(L.keys2 + n * 4);
  L.vals2 = align256(L.vals + n * 8);
  L.temp = align256(L.vals2 + n * 8);
  L.temp_bytes = 0;
  int end_bit = 1;
  while ((1ull << end_bit) < (uint64_t)n_cells + 2) ++end_bit;
  cub::DoubleBuffer<uint32_t> dk(nullptr, nullptr);
  cub::DoubleBuffer<unsigned long long> dv(nullptr, nullptr);
  cub::DeviceRadixSort::SortPairs(nullptr, L.temp_bytes, dk, dv, (int)n, 0, end_bit);
  L.total = align256(L.temp + L.temp_bytes);
  return L;
}

}  // namespace

bool ingest_sorted_fits(uint64_t n) { return n >= 1 && n < (1ull << 31); }

size_t ingest_sort_tmp_bytes(uint64_t n, uint32_t n_cells) { return sort_layout(n, n_cells).total; }

cudaError_t launch_ingest_sorted_keys(const uint4* upd, uint64_t n, const DevGraph& g, const DevState& s,
                                      void* tmp, SortedBatch* out, cudaStream_t st) {
  const SortLayout L = sort_layout(n, g.n_cells);
  char* base = static_cast<char*>(tmp);
  uint32_t* keys = reinterpret_cast<uint32_t*>(base + L.keys);
  unsigned long long* vals = reinterpret_cast<unsigned long long*>(base + L.vals);
  const unsigned blocks = (unsigned)((n + ST - 1) / ST);
  k_bulk_keys<<<(unsigned)((n + ST * KPT - 1) / (ST * KPT)), ST, 0, st>>>(upd, n, g, s, keys, vals);
  int end_bit = 1;
  while ((1ull << end_bit) < (uint64_t)g.n_cells + 2) ++end_bit;
  cub::DoubleBuffer<uint32_t> dk(keys, reinterpret_cast<uint32_t*>(base + L.keys2));
  cub::DoubleBuffer<unsigned long long> dv(vals, reinterpret_cast<unsigned long long*>(base + L.vals2));
  size_t tb = L.temp_bytes;
  const cudaError_t e = cub::DeviceRadixSort::SortPairs(base + L.temp, tb, dk, dv, (int)n, 0, end_bit, st);
  if (e != cudaSuccess) return e;
  k_bulk_runs<<<blocks, ST, 0, st>>>(dk.Current(), n, g, s);
  out->keys = dk.Current();  // (where the sort left the ordered pairs: decided on the host)
  out->vals = dv.Current();
  return cudaGetLastError();
}

void launch_ingest_sorted_scatter(const uint4* upd, uint64_t n, uint32_t seq0, const DevGraph& g,
                                  const DevState& s, const SortedBatch& b, cudaStream_t st) {
  k_bulk_scatter<<<(unsigned)((n + ST * SPT - 1) / (ST * SPT)), ST, 0, st>>>(upd, b.keys, b.vals, n, seq0, g, s);
}

}  // namespace gg

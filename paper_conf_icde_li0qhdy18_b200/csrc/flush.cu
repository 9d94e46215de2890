// flush.cu — message cleaning of a set of cells (Alg. 2 steps 3-4, P@22374-23566).
//
// The paper copies the cells' buckets over PCIe, runs one thread per bucket with a warp
// X-shuffle into a per-object intermediate table T (Alg. 3, P@24850) and a GPU_Collect
// pass building R[c] (P@23070-23566), then ships R back to the CPU.  That design is prior
// art (north_star); here one CTA owns one cell and streams its log once:
//
//  phase A/B  per tile of 4 records/thread (128-bit loads of obj, 2x128-bit of keys),
//             tiles newest-first so the first record seen per object is usually its
//             newest: a shared-memory open-addressing table obj -> max key (atomicMax
//             only when the key beats the stored one) and, after a barrier, the position
//             of the record holding that max (per-object segmented arg-max on (t, seq)).
//  phase C    winners are valid iff key == ot_key[obj] (one gather per distinct object;
//             replaces tombstones, reading R8/R9); counts per source vertex in smem.
//  phase D    block scan -> per-vertex offsets, one bump allocation of the compacted
//             list R[c] (sorted by source vertex) in the arena, v_obj[v] = (start, n),
//             scatter of the winners' payload, cell marked clean.
// If a cell holds more distinct objects than the table, the CTA falls back to a two-pass
// filter (key == ot_key[obj] per record) for that cell.
#include "internal.cuh"

namespace gg {

namespace {
constexpr int FT = 512;               // threads per CTA
constexpr int TCAP = 2048;            // table slots (power of two)
constexpr int HCAP = 4096;            // per-vertex counters kept in smem
constexpr int RPT = 4;                // records per thread per tile
constexpr int TILE = FT * RPT;
constexpr int MAX_PROBE = 64;

struct FlushSmem {
  uint32_t tab_obj[TCAP];
  unsigned long long tab_key[TCAP];
  uint32_t tab_pos[TCAP];
  uint32_t hist[HCAP];
  uint32_t wsum[FT / 32];
  uint32_t idx;
  uint32_t n_valid;
  int overflow;
  int fail;
  unsigned long long out;
  unsigned long long nrec;
};

__device__ __forceinline__ uint32_t hslot(uint32_t o) { return (o * 2654435761u) >> (32 - 11); }
static_assert(TCAP == 2048, "hslot assumes 2^11 slots");

__device__ __forceinline__ int tab_find_insert(uint32_t* tab_obj, uint32_t o) {
  uint32_t h = hslot(o);
  volatile uint32_t* vt = tab_obj;
#pragma unroll 1
  for (int p = 0; p < MAX_PROBE; ++p) {
    uint32_t s = (h + p) & (TCAP - 1);
    uint32_t cur = vt[s];
    if (cur == o) return (int)s;
    if (cur == NONE) {
      uint32_t old = atomicCAS(&tab_obj[s], NONE, o);
      if (old == NONE || old == o) return (int)s;
    }
  }
  return -1;
}

// In-place exclusive scan of a[0..n) (smem or global) by the whole CTA; returns the total.
__device__ uint32_t block_exclusive_scan(uint32_t* a, uint32_t n, uint32_t* wsum) {
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  uint32_t carry = 0;
  for (uint32_t base = 0; base < n; base += FT) {
    uint32_t i = base + tid;
    uint32_t v = i < n ? a[i] : 0;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) wsum[wid] = x;
    __syncthreads();
    if (wid == 0) {
      uint32_t t = lane < FT / 32 ? wsum[lane] : 0;
#pragma unroll
      for (int o = 1; o < FT / 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xffffffffu, t, o);
        if (lane >= o) t += y;
      }
      if (lane < FT / 32) wsum[lane] = t;  // inclusive warp totals
    }
    __syncthreads();
    uint32_t wpre = wid ? wsum[wid - 1] : 0;
    if (i < n) a[i] = carry + wpre + x - v;
    uint32_t tot = wsum[FT / 32 - 1];
    __syncthreads();
    carry += tot;
  }
  return carry;
}

struct Seg {
  uint32_t start, len;
};

__global__ void __launch_bounds__(FT) k_flush(DevGraph g, DevState s, Arena out,
                                              unsigned long long* out_top, uint32_t begin,
                                              uint2* cell_comp, uint32_t* vcnt_global) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  FlushSmem& sm = *reinterpret_cast<FlushSmem*>(smem_raw);
  const int tid = threadIdx.x;
  DevStatus* st = s.st;

  for (;;) {
    if (tid == 0) sm.idx = begin + atomicAdd(&st->flush_work, 1u);
    __syncthreads();
    const uint32_t li = sm.idx;
    const uint32_t lend = *((volatile unsigned*)&st->n_flush);
    if (blockIdx.x == 0 && tid == 0) st->flush_end = lend;
    if (li >= lend) break;
    const uint32_t c = s.flush_list[li];
    const uint32_t head = s.cell_head[c];
    const uint2 comp = cell_comp[c];
    const uint32_t cbeg = c * g.cs;
    const uint32_t nvert = min(g.cs, g.V - cbeg);
    uint32_t* cnt = (nvert <= (uint32_t)HCAP) ? sm.hist : (vcnt_global + cbeg);

    // --- phase A/B: per-object arg-max over the cell's records, newest extent first ---
    for (int i = tid; i < TCAP; i += FT) {
      sm.tab_obj[i] = NONE;
      sm.tab_key[i] = 0ull;
    }
    if (tid == 0) {
      sm.overflow = 0;
      sm.fail = 0;
      sm.n_valid = 0;
      sm.nrec = 0;
    }
    __syncthreads();
    uint32_t e = head;
    unsigned long long nrec = 0;
    // segments: pending extents newest-first, then the previous compacted list
    for (;;) {
      Seg sg;
      uint32_t enext = NONE;
      if (e != NONE) {
        sg.start = s.x_start[e];
        sg.len = s.x_len[e];
        enext = s.x_next[e];
      } else {
        sg.start = comp.x;
        sg.len = comp.y;
      }
      nrec += sg.len;
      const int ntiles = (int)((sg.len + TILE - 1) / TILE);
      for (int t = ntiles - 1; t >= 0; --t) {
        const uint32_t rb = (uint32_t)t * TILE + (uint32_t)tid * RPT;
        uint32_t o[RPT] = {0, 0, 0, 0};
        unsigned long long k[RPT] = {0, 0, 0, 0};
        int slot[RPT];
        bool ok[RPT];
        if (rb < sg.len) {
          const uint4 o4 = __ldg(reinterpret_cast<const uint4*>(s.ar.obj + sg.start + rb));
          const ulonglong2 k01 = __ldg(reinterpret_cast<const ulonglong2*>(s.ar.key + sg.start + rb));
          const ulonglong2 k23 = __ldg(reinterpret_cast<const ulonglong2*>(s.ar.key + sg.start + rb + 2));
          o[0] = o4.x; o[1] = o4.y; o[2] = o4.z; o[3] = o4.w;
          k[0] = k01.x; k[1] = k01.y; k[2] = k23.x; k[3] = k23.y;
        }
#pragma unroll
        for (int j = 0; j < RPT; ++j) {
          ok[j] = rb + j < sg.len;
          slot[j] = -1;
          if (ok[j]) {
            slot[j] = tab_find_insert(sm.tab_obj, o[j]);
            if (slot[j] < 0) {
              sm.overflow = 1;
            } else if (k[j] > ((volatile unsigned long long*)sm.tab_key)[slot[j]]) {
              atomicMax(&sm.tab_key[slot[j]], k[j]);
            }
          }
        }
        __syncthreads();
#pragma unroll
        for (int j = 0; j < RPT; ++j)
          if (slot[j] >= 0 && k[j] == sm.tab_key[slot[j]]) sm.tab_pos[slot[j]] = sg.start + rb + j;
        __syncthreads();
      }
      if (e == NONE) break;
      e = enext;
    }
    const bool overflow = sm.overflow != 0;

    // --- phase C: validity (key == ot_key) and per-vertex counts ---
    for (uint32_t i = tid; i < nvert; i += FT) cnt[i] = 0;
    __syncthreads();
    if (!overflow) {
      for (int i = tid; i < TCAP; i += FT) {
        const uint32_t ob = sm.tab_obj[i];
        if (ob == NONE) continue;
        if (sm.tab_key[i] == s.ot_key[ob]) {
          atomicAdd(&cnt[s.ar.vsrc[sm.tab_pos[i]] - cbeg], 1u);
          atomicAdd(&sm.n_valid, 1u);
        } else {
          sm.tab_obj[i] = NONE;  // stale: the object's latest update is elsewhere
        }
      }
    } else {
      // filter fallback, pass 1: every record, valid iff key == ot_key[obj]
      uint32_t e2 = head;
      for (;;) {
        Seg sg;
        uint32_t enext = NONE;
        if (e2 != NONE) {
          sg.start = s.x_start[e2];
          sg.len = s.x_len[e2];
          enext = s.x_next[e2];
        } else {
          sg.start = comp.x;
          sg.len = comp.y;
        }
        for (uint32_t r = tid; r < sg.len; r += FT) {
          const uint32_t p = sg.start + r;
          const uint32_t ob = s.ar.obj[p];
          if (s.ar.key[p] == s.ot_key[ob]) {
            atomicAdd(&cnt[s.ar.vsrc[p] - cbeg], 1u);
            atomicAdd(&sm.n_valid, 1u);
          }
        }
        if (e2 == NONE) break;
        e2 = enext;
      }
    }
    __syncthreads();
    block_exclusive_scan(cnt, nvert, sm.wsum);
    if (tid == 0) {
      const unsigned long long alloc = (sm.n_valid + 3u) & ~3ull;
      const unsigned long long o0 = atomicAdd(out_top, alloc);
      sm.out = o0;
      if (o0 + alloc > out.cap) {
        sm.fail = 1;
        atomicOr(&st->err, (unsigned)ERR_ARENA);
      }
    }
    __syncthreads();
    if (!sm.fail) {
      const unsigned long long ob0 = sm.out;
      const uint32_t nv = sm.n_valid;
      for (uint32_t i = tid; i < nvert; i += FT) {
        const uint32_t b = cnt[i];
        const uint32_t en = (i + 1 < nvert) ? cnt[i + 1] : nv;
        s.v_obj[cbeg + i] = make_uint2((uint32_t)(ob0 + b), en - b);
      }
      __syncthreads();
      // --- phase D: scatter the winners (payload gathered from their record) ---
      if (!overflow) {
        for (int i = tid; i < TCAP; i += FT) {
          const uint32_t ob = sm.tab_obj[i];
          if (ob == NONE) continue;
          const uint32_t p = sm.tab_pos[i];
          const uint32_t vs = s.ar.vsrc[p];
          const uint32_t q = (uint32_t)ob0 + atomicAdd(&cnt[vs - cbeg], 1u);
          out.obj[q] = ob;
          out.key[q] = sm.tab_key[i];
          out.vsrc[q] = vs;
          out.off[q] = s.ar.off[p];
          out.edge[q] = s.ar.edge[p];
        }
      } else {
        uint32_t e2 = head;
        for (;;) {
          Seg sg;
          uint32_t enext = NONE;
          if (e2 != NONE) {
            sg.start = s.x_start[e2];
            sg.len = s.x_len[e2];
            enext = s.x_next[e2];
          } else {
            sg.start = comp.x;
            sg.len = comp.y;
          }
          for (uint32_t r = tid; r < sg.len; r += FT) {
            const uint32_t p = sg.start + r;
            const uint32_t ob = s.ar.obj[p];
            const unsigned long long kk = s.ar.key[p];
            if (kk == s.ot_key[ob]) {
              const uint32_t vs = s.ar.vsrc[p];
              const uint32_t q = (uint32_t)ob0 + atomicAdd(&cnt[vs - cbeg], 1u);
              out.obj[q] = ob;
              out.key[q] = kk;
              out.vsrc[q] = vs;
              out.off[q] = s.ar.off[p];
              out.edge[q] = s.ar.edge[p];
            }
          }
          if (e2 == NONE) break;
          e2 = enext;
        }
      }
      __syncthreads();
      if (tid == 0) {
        cell_comp[c] = make_uint2((uint32_t)ob0, nv);
        s.cell_head[c] = NONE;
        s.cell_pending[c] = 0;
        atomicAdd(&st->records_flushed, nrec);
        atomicAdd(&st->objects_written, (unsigned long long)nv);
        atomicAdd(&st->cells_flushed, 1ull);
      }
    }
    __syncthreads();
  }
}

int g_flush_blocks_per_sm = 0;
}  // namespace

int flush_smem_bytes() { return (int)sizeof(FlushSmem); }

void launch_flush(const DevGraph& g, const DevState& s, const Arena& out,
                  unsigned long long* out_top, uint32_t begin, int sm_count, cudaStream_t st) {
  const int smem = (int)sizeof(FlushSmem);
  if (g_flush_blocks_per_sm == 0) {
    cudaFuncSetAttribute(k_flush, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    int b = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_flush, FT, smem);
    g_flush_blocks_per_sm = b > 0 ? b : 1;
  }
  const int grid = sm_count * g_flush_blocks_per_sm;
  k_flush<<<grid, FT, smem, st>>>(g, s, out, out_top, begin, s.cell_comp, s.vcnt);
}

}  // namespace gg

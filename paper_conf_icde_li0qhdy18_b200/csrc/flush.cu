// flush.cu — message cleaning of a set of cells (Alg. 2 steps 3-4, P@22374-23566).
//
// The paper copies the cells' buckets over PCIe, runs one thread per bucket with a warp
// X-shuffle into a per-object intermediate table T (Alg. 3, P@24850) and a GPU_Collect
// pass building R[c] (P@23070-23566), then ships R back to the CPU.  That design is prior
// art (north_star); here one CTA owns one cell at a time and streams its log once:
//
//  gather     the cell's extents (newest first, then its previous cleaned list) into a
//             shared-memory list; the extents form one logical record sequence, tiled
//             across extent boundaries (extents start on 4-record boundaries, so every
//             4-record group is one 128-bit load of obj and two of keys); the next tile's
//             loads are issued before the current tile is processed.
//  phase A/B  per tile: shared-memory open-addressing table keyed by obj.  The per-object
//             arg-max on (t, seq) is already resolved by ingest, which RED.MAX-es every key
//             into ot_key[obj] (native 64-bit global atomics; shared memory has no 64-bit
//             max, only a CAS spin loop that collapses under contention).  So the thread
//             that first inserts an object caches its target ot_key[obj] in the table (one
//             gather per distinct object per cell), and after a barrier the record whose key
//             equals the target records its position.  Objects whose newest record lives in
//             another cell match nothing and are dropped (replaces tombstones, R8/R9).
//  phase C    counts of the matched objects per source vertex.
//  phase D    block scan -> per-vertex offsets, one bump allocation of the cleaned list
//             R[c] (sorted by source vertex), v_obj[v] = (start, n), payload scatter, the
//             cell marked clean.
// A cell holding more distinct objects than the table falls back to a two-pass filter.
// The table size is chosen per launch from the live objects per cell.
#include "internal.cuh"

namespace gg {

namespace {
constexpr int FT = 128;        // threads per CTA (8 CTAs per SM)
constexpr int RPT = 4;         // records per thread per tile (one 128-bit load of obj)
constexpr int TILE = FT * RPT;
constexpr int XMAX = 32;       // extents gathered per pass over the chain
constexpr int MAX_PROBE = 64;

template <int TCAP, int HCAP>
struct FlushSmem {
  uint32_t tab_obj[TCAP];
  unsigned long long tab_tgt[TCAP];  // ot_key[obj]: the object's newest (t<<32|seq)
  uint32_t tab_pos[TCAP];            // arena position of the record holding it, or NONE
  uint32_t hist[HCAP];
  uint32_t xs[XMAX];
  uint32_t xl[XMAX];
  uint32_t xpre[XMAX + 1];
  uint32_t wsum[FT / 32];
  uint32_t nx;
  uint32_t e_next;
  uint32_t idx;
  uint32_t n_valid;
  int overflow;
  int fail;
  int comp_done;
  unsigned long long out;
};

template <int TCAP>
__device__ __forceinline__ int tab_find_insert(uint32_t* tab_obj, uint32_t o, bool& inserted) {
  constexpr int BITS = __builtin_ctz(TCAP);
  uint32_t h = (o * 2654435761u) >> (32 - BITS);
  volatile uint32_t* vt = tab_obj;
  inserted = false;
#pragma unroll 1
  for (int p = 0; p < MAX_PROBE; ++p) {
    const uint32_t cur = vt[h];
    if (cur == o) return (int)h;
    if (cur == NONE) {
      const uint32_t old = atomicCAS(&tab_obj[h], NONE, o);
      if (old == NONE) {
        inserted = true;
        return (int)h;
      }
      if (old == o) return (int)h;
    }
    h = (h + 1) & (TCAP - 1);
  }
  return -1;
}

// In-place exclusive scan of a[0..n) (smem or global) by the whole CTA, RPT items per
// thread per pass; returns the total.
__device__ uint32_t block_exclusive_scan(uint32_t* a, uint32_t n, uint32_t* wsum) {
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  uint32_t carry = 0;
  for (uint32_t base = 0; base < n; base += FT * RPT) {
    uint32_t v[RPT];
    uint32_t loc = 0;
#pragma unroll
    for (int j = 0; j < RPT; ++j) {
      const uint32_t i = base + tid * RPT + j;
      v[j] = i < n ? a[i] : 0;
      loc += v[j];
    }
    uint32_t x = loc;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) wsum[wid] = x;
    __syncthreads();
    if (wid == 0) {
      uint32_t t = lane < FT / 32 ? wsum[lane] : 0;
#pragma unroll
      for (int o = 1; o < FT / 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, t, o);
        if (lane >= o) t += y;
      }
      if (lane < FT / 32) wsum[lane] = t;
    }
    __syncthreads();
    uint32_t run = carry + (wid ? wsum[wid - 1] : 0) + x - loc;
#pragma unroll
    for (int j = 0; j < RPT; ++j) {
      const uint32_t i = base + tid * RPT + j;
      if (i < n) a[i] = run;
      run += v[j];
    }
    const uint32_t tot = wsum[FT / 32 - 1];
    __syncthreads();
    carry += tot;
  }
  return carry;
}

// Gather up to XMAX segments of cell c's log starting at chain extent e (the cleaned list
// goes last).  Thread 0 walks; the list is published in shared memory.
template <class SM>
__device__ void gather_extents(SM& sm, const DevState& s, uint32_t e, uint2 comp) {
  if (threadIdx.x == 0) {
    uint32_t n = 0, pre = 0;
    while (e != NONE && n < XMAX) {
      const uint32_t st = s.x_start[e], ln = s.x_len[e];
      const uint32_t nxt = s.x_next[e];
      sm.xs[n] = st;
      sm.xl[n] = ln;
      sm.xpre[n] = pre;
      pre += (ln + 3u) & ~3u;
      ++n;
      e = nxt;
    }
    sm.comp_done = 0;
    if (e == NONE && n < XMAX) {
      if (comp.y) {
        sm.xs[n] = comp.x;
        sm.xl[n] = comp.y;
        sm.xpre[n] = pre;
        pre += (comp.y + 3u) & ~3u;
        ++n;
      }
      sm.comp_done = 1;
    }
    sm.xpre[n] = pre;
    sm.nx = n;
    sm.e_next = e;
  }
  __syncthreads();
}

struct Grp {
  uint4 o;
  ulonglong2 k01, k23;
  uint32_t pos;   // arena position of the group's first record
  uint32_t nv;    // valid records in the group (0..4)
};

template <class SM>
__device__ __forceinline__ Grp load_group(const SM& sm, const DevState& s, uint32_t L, int& j) {
  Grp r;
  r.nv = 0;
  r.pos = 0;
  if (L >= sm.xpre[sm.nx]) return r;
  while (j + 1 < (int)sm.nx && sm.xpre[j + 1] <= L) ++j;  // L only grows: j only advances
  // each extent is read back to front (records are appended in arrival order), so an
  // object's newest record tends to be seen first and later ones rarely need an atomic
  const uint32_t ro = (sm.xpre[j + 1] - sm.xpre[j]) - 4u - (L - sm.xpre[j]);
  r.pos = sm.xs[j] + ro;
  const uint32_t len = sm.xl[j];
  r.nv = ro >= len ? 0 : min(4u, len - ro);
  if (r.nv) {
    r.o = __ldg(reinterpret_cast<const uint4*>(s.ar.obj + r.pos));
    r.k01 = __ldg(reinterpret_cast<const ulonglong2*>(s.ar.key + r.pos));
    r.k23 = __ldg(reinterpret_cast<const ulonglong2*>(s.ar.key + r.pos + 2));
  }
  return r;
}

template <int TCAP, int HCAP>
__global__ void __launch_bounds__(FT, 8) k_flush(DevGraph g, DevState s, Arena out,
                                                 unsigned long long* out_top, uint32_t begin) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  using SM = FlushSmem<TCAP, HCAP>;
  SM& sm = *reinterpret_cast<SM*>(smem_raw);
  const int tid = threadIdx.x;
  DevStatus* st = s.st;
  const uint32_t lend = *((volatile unsigned*)&st->n_flush);
  if (blockIdx.x == 0 && tid == 0) st->flush_end = lend;
  const uint32_t G = gridDim.x;

  // Static schedule (cells li = begin + blockIdx.x + i*G) so the next cells' metadata can
  // be loaded a cell ahead: cell id two ahead, (head, comp) one ahead, consumed next turn.
  uint32_t li = begin + blockIdx.x;
  uint32_t c = li < lend ? s.flush_list[li] : 0;
  uint32_t head = li < lend ? s.cell_head[c] : NONE;
  uint2 comp = li < lend ? s.cell_comp[c] : make_uint2(0, 0);
  uint32_t c_n = li + G < lend ? s.flush_list[li + G] : 0;
  for (; li < lend; li += G) {
    uint32_t head_n = NONE, c_nn = 0;
    uint2 comp_n = make_uint2(0, 0);
    if (li + G < lend) {
      head_n = s.cell_head[c_n];
      comp_n = s.cell_comp[c_n];
    }
    if (li + 2 * G < lend) c_nn = s.flush_list[li + 2 * G];
    const uint32_t cbeg = c * g.cs;
    const uint32_t nvert = min(g.cs, g.V - cbeg);
    uint32_t* cnt = (nvert <= (uint32_t)HCAP) ? sm.hist : (s.vcnt + cbeg);

    for (int i = tid; i < TCAP; i += FT) {
      sm.tab_obj[i] = NONE;
      sm.tab_pos[i] = NONE;
    }
    if (tid == 0) {
      sm.overflow = 0;
      sm.fail = 0;
      sm.n_valid = 0;
    }
    // ---- phase A/B over the log, XMAX extents at a time ------------------------------------
    unsigned long long nrec = 0;
    uint32_t e = head;
    for (;;) {
      __syncthreads();
      gather_extents(sm, s, e, comp);
      const uint32_t total = sm.xpre[sm.nx];
      for (uint32_t j = 0; j < sm.nx; ++j) nrec += sm.xl[j];
      const uint32_t ntiles = (total + TILE - 1) / TILE;
      // One barrier per tile: [A(t)] bar [B(t) A(t+1)] bar [B(t+1) A(t+2)] ...  B(t) may race
      // with A(t+1) raising a maximum; then the newer record writes its position in B(t+1),
      // after the next barrier, so the last position written is always the maximum's.
      int xj = 0;
      Grp cur = load_group(sm, s, (uint32_t)tid * RPT, xj);
      uint32_t o[RPT];
      unsigned long long k[RPT];
      int slot[RPT];
      auto phase_a = [&](const Grp& gr) {
        o[0] = gr.o.x; o[1] = gr.o.y; o[2] = gr.o.z; o[3] = gr.o.w;
        k[0] = gr.k01.x; k[1] = gr.k01.y; k[2] = gr.k23.x; k[3] = gr.k23.y;
#pragma unroll
        for (int j = RPT - 1; j >= 0; --j) {  // newest record of the group first
          slot[j] = -1;
          if ((uint32_t)j < gr.nv) {
            bool ins;
            slot[j] = tab_find_insert<TCAP>(sm.tab_obj, o[j], ins);
            if (slot[j] < 0) {
              sm.overflow = 1;
            } else if (ins) {
              sm.tab_tgt[slot[j]] = s.ot_key[o[j]];  // first sight: cache the target
            }
          }
        }
      };
      if (ntiles) phase_a(cur);
      for (uint32_t t = 0; t < ntiles; ++t) {
        Grp nxt;
        nxt.nv = 0;
        if (t + 1 < ntiles) nxt = load_group(sm, s, (t + 1) * TILE + (uint32_t)tid * RPT, xj);
        __syncthreads();
#pragma unroll
        for (int j = 0; j < RPT; ++j)
          if (slot[j] >= 0 && k[j] == sm.tab_tgt[slot[j]]) sm.tab_pos[slot[j]] = cur.pos + j;
        if (t + 1 < ntiles) {
          cur = nxt;
          phase_a(cur);
        }
      }
      __syncthreads();
      if (sm.comp_done) break;
      e = sm.e_next;
    }
    const bool overflow = sm.overflow != 0;

    // ---- phase C: validity (key == ot_key) and per-vertex counts ----------------------------
    for (uint32_t i = tid; i < nvert; i += FT) cnt[i] = 0;
    __syncthreads();
    if (!overflow) {
      for (int i = tid; i < TCAP; i += FT) {
        const uint32_t ob = sm.tab_obj[i];
        if (ob == NONE) continue;
        if (sm.tab_pos[i] != NONE) {
          atomicAdd(&cnt[s.ar.vsrc[sm.tab_pos[i]] - cbeg], 1u);
          atomicAdd(&sm.n_valid, 1u);
        } else {
          sm.tab_obj[i] = NONE;  // stale: the object's latest update is elsewhere
        }
      }
    } else {
      // filter fallback, pass 1: every record, valid iff key == ot_key[obj]
      uint32_t e2 = head;
      bool last = false;
      while (!last) {
        uint32_t sst, sln;
        if (e2 != NONE) {
          sst = s.x_start[e2];
          sln = s.x_len[e2];
          e2 = s.x_next[e2];
        } else {
          sst = comp.x;
          sln = comp.y;
          last = true;
        }
        for (uint32_t r = tid; r < sln; r += FT) {
          const uint32_t p = sst + r;
          const uint32_t ob = s.ar.obj[p];
          if (s.ar.key[p] == s.ot_key[ob]) {
            atomicAdd(&cnt[s.ar.vsrc[p] - cbeg], 1u);
            atomicAdd(&sm.n_valid, 1u);
          }
        }
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
      // ---- phase D: scatter the winners (payload gathered from their record) ----------------
      if (!overflow) {
        for (int i = tid; i < TCAP; i += FT) {
          const uint32_t ob = sm.tab_obj[i];
          if (ob == NONE) continue;
          const uint32_t p = sm.tab_pos[i];
          const uint32_t vs = s.ar.vsrc[p];
          const uint32_t q = (uint32_t)ob0 + atomicAdd(&cnt[vs - cbeg], 1u);
          out.obj[q] = ob;
          out.key[q] = sm.tab_tgt[i];
          out.vsrc[q] = vs;
          out.off[q] = s.ar.off[p];
          out.edge[q] = s.ar.edge[p];
        }
      } else {
        uint32_t e2 = head;
        bool last = false;
        while (!last) {
          uint32_t sst, sln;
          if (e2 != NONE) {
            sst = s.x_start[e2];
            sln = s.x_len[e2];
            e2 = s.x_next[e2];
          } else {
            sst = comp.x;
            sln = comp.y;
            last = true;
          }
          for (uint32_t r = tid; r < sln; r += FT) {
            const uint32_t p = sst + r;
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
        }
      }
      __syncthreads();
      if (tid == 0) {
        s.cell_comp[c] = make_uint2((uint32_t)ob0, nv);
        s.cell_head[c] = NONE;
        s.cell_pending[c] = 0;
        atomicAdd(&st->objects_written, (unsigned long long)nv);
        atomicAdd(&st->cells_flushed, 1ull);
      }
    }
    if (tid == 0 && !sm.fail) atomicAdd(&st->records_flushed, nrec);
    __syncthreads();
    c = c_n;
    head = head_n;
    comp = comp_n;
    c_n = c_nn;
  }
}

template <int TCAP, int HCAP>
void launch_t(const DevGraph& g, const DevState& s, const Arena& out, unsigned long long* out_top,
              uint32_t begin, int sm_count, cudaStream_t st) {
  static int blocks_per_sm = 0;
  const int smem = (int)sizeof(FlushSmem<TCAP, HCAP>);
  if (blocks_per_sm == 0) {
    cudaFuncSetAttribute(k_flush<TCAP, HCAP>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    int b = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_flush<TCAP, HCAP>, FT, smem);
    blocks_per_sm = b > 0 ? b : 1;
  }
  k_flush<TCAP, HCAP><<<sm_count * blocks_per_sm, FT, smem, st>>>(g, s, out, out_top, begin);
}
}  // namespace

void launch_flush(const DevGraph& g, const DevState& s, const Arena& out,
                  unsigned long long* out_top, uint32_t begin, uint32_t objects_per_cell,
                  int sm_count, cudaStream_t st) {
  // table sized for ~4x the live objects of an average cell (overflow falls back safely)
  const bool small_t = objects_per_cell <= 64;
  const bool small_h = g.cs <= 1024;
  if (small_t && small_h) launch_t<256, 1024>(g, s, out, out_top, begin, sm_count, st);
  else if (small_t) launch_t<256, 4096>(g, s, out, out_top, begin, sm_count, st);
  else if (small_h) launch_t<2048, 1024>(g, s, out, out_top, begin, sm_count, st);
  else launch_t<2048, 4096>(g, s, out, out_top, begin, sm_count, st);
}

}  // namespace gg

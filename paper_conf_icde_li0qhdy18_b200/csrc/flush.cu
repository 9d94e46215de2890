// flush.cu — message cleaning of a set of cells (Alg. 2 steps 3-4, P@22374-23566).
//
// The paper copies the cells' buckets over PCIe, runs one thread per bucket with a warp
// X-shuffle into a per-object intermediate table T (Alg. 3, P@24850) and a GPU_Collect
// pass building R[c] (P@23070-23566), then ships R back to the CPU.  That design is prior
// art (north_star).  Here the per-object arg-max on (t, seq) is split in two:
//
//   ingest   RED.MAX-es every message's key (t<<32 | seq) into ot_key[obj] (native 64-bit
//            global atomics, csrc/ingest.cu) — the object table of P@15869 holding the max;
//   flush    streams the cell's log once and keeps, per object, the one record whose key
//            equals ot_key[obj] (keys are unique, so exactly one record in the whole log
//            matches; if it lives in another cell the object has moved away: no tombstones
//            are needed, readings R8/R9).
//
// One CTA cleans one cell at a time (static schedule, the next cells' metadata loaded a
// cell ahead):
//   gather   the cell's extents (newest first, then its previous cleaned list) into a
//            shared-memory list; they form one logical record sequence tiled across extent
//            boundaries (extents start on 4-record boundaries: every 4-record group is one
//            128-bit load of obj and two of keys).  Each warp streams its own groups with
//            the next group's loads in flight; no barrier inside the stream.
//   match    per record: ot_key[obj] through L1 (a cell touches a few dozen objects, so
//            the lines stay resident), compare; matches are appended to a shared winner list.
//   index    counts per source vertex, block scan, one bump allocation of the cleaned list
//            R[c] (sorted by source vertex), v_obj[v] = (start, n), payload scatter, the
//            cell marked clean.
// A cell with more winners than the shared list falls back to a second streaming pass.
#include "internal.cuh"

namespace gg {

namespace {
constexpr int FT = 128;        // threads per CTA (8 CTAs per SM)
constexpr int NW = FT / 32;
constexpr int RPT = 4;         // records per lane per group (one 128-bit load of obj)
constexpr int XMAX = 32;       // extents gathered per pass over the chain
constexpr int WCAP = 2048;     // winners kept in shared memory

template <int HCAP>
struct FlushSmem {
  uint32_t win[WCAP];  // arena positions of the matched records
  uint32_t hist[HCAP];
  uint32_t xs[XMAX];
  uint32_t xl[XMAX];
  uint32_t xpre[XMAX + 1];
  uint32_t wsum[NW];
  uint32_t nx;
  uint32_t e_next;
  uint32_t n_win;
  int comp_done;
  int fail;
  unsigned long long out;
};

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
      uint32_t t = lane < NW ? wsum[lane] : 0;
#pragma unroll
      for (int o = 1; o < NW; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, t, o);
        if (lane >= o) t += y;
      }
      if (lane < NW) wsum[lane] = t;
    }
    __syncthreads();
    uint32_t run = carry + (wid ? wsum[wid - 1] : 0) + x - loc;
#pragma unroll
    for (int j = 0; j < RPT; ++j) {
      const uint32_t i = base + tid * RPT + j;
      if (i < n) a[i] = run;
      run += v[j];
    }
    const uint32_t tot = wsum[NW - 1];
    __syncthreads();
    carry += tot;
  }
  return carry;
}

// Gather up to XMAX segments of the cell's log starting at chain extent e (the previous
// cleaned list goes last).  Thread 0 walks; the list is published in shared memory.
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
  uint32_t pos;  // arena position of the group's first record
  uint32_t nv;   // valid records in the group (0..4)
};

// The 4-record group at logical offset L (a multiple of 4).  j is the lane's extent cursor
// (L only grows along a lane's stream, so j only advances).
template <class SM>
__device__ __forceinline__ Grp load_group(const SM& sm, const DevState& s, uint32_t L, int& j) {
  Grp r;
  r.nv = 0;
  r.pos = 0;
  if (L >= sm.xpre[sm.nx]) return r;
  while (j + 1 < (int)sm.nx && sm.xpre[j + 1] <= L) ++j;
  const uint32_t off = L - sm.xpre[j];
  r.pos = sm.xs[j] + off;
  const uint32_t len = sm.xl[j];
  r.nv = off >= len ? 0 : min(4u, len - off);
  if (r.nv) {
    r.o = __ldg(reinterpret_cast<const uint4*>(s.ar.obj + r.pos));
    r.k01 = __ldg(reinterpret_cast<const ulonglong2*>(s.ar.key + r.pos));
    r.k23 = __ldg(reinterpret_cast<const ulonglong2*>(s.ar.key + r.pos + 2));
  }
  return r;
}

template <int HCAP>
__global__ void __launch_bounds__(FT, 8) k_flush(DevGraph g, DevState s, Arena out,
                                                 unsigned long long* out_top, uint32_t begin) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  using SM = FlushSmem<HCAP>;
  SM& sm = *reinterpret_cast<SM*>(smem_raw);
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const unsigned lt = lanemask_lt();
  DevStatus* st = s.st;
  const uint32_t lend = *((volatile unsigned*)&st->n_flush);
  if (blockIdx.x == 0 && tid == 0) st->flush_end = lend;
  const uint32_t G = gridDim.x;
  const unsigned long long* __restrict__ otk = s.ot_key;

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
    if (tid == 0) {
      sm.n_win = 0;
      sm.fail = 0;
    }

    // ---- match: stream the log, keep the record equal to ot_key[obj] ---------------------
    unsigned long long nrec = 0;
    uint32_t e = head;
    for (;;) {
      __syncthreads();
      gather_extents(sm, s, e, comp);
      const uint32_t total = sm.xpre[sm.nx];
      if (tid == 0)
        for (uint32_t j = 0; j < sm.nx; ++j) nrec += sm.xl[j];
      // warp w takes groups of 32*RPT records: L = (w + NW*i) * 128 + lane * 4
      int xj = 0;
      uint32_t L = (uint32_t)wid * (32 * RPT) + (uint32_t)lane * RPT;
      Grp cur = load_group(sm, s, L, xj);
      while (__any_sync(0xffffffffu, L < total)) {
        const uint32_t Ln = L + NW * 32 * RPT;
        const Grp nxt = load_group(sm, s, Ln, xj);
        const uint32_t o[RPT] = {cur.o.x, cur.o.y, cur.o.z, cur.o.w};
        const unsigned long long k[RPT] = {cur.k01.x, cur.k01.y, cur.k23.x, cur.k23.y};
#pragma unroll
        for (int j = 0; j < RPT; ++j) {
          const bool hit = (uint32_t)j < cur.nv && __ldg(otk + o[j]) == k[j];
          const unsigned hm = __ballot_sync(0xffffffffu, hit);
          if (hm) {
            uint32_t base = 0;
            if (lane == __ffs(hm) - 1) base = atomicAdd(&sm.n_win, (unsigned)__popc(hm));
            base = __shfl_sync(0xffffffffu, base, __ffs(hm) - 1);
            const uint32_t w = base + __popc(hm & lt);
            if (hit && w < WCAP) sm.win[w] = cur.pos + j;
          }
        }
        cur = nxt;
        L = Ln;
      }
      __syncthreads();
      if (sm.comp_done) break;
      e = sm.e_next;
    }
    const uint32_t n_win = sm.n_win;
    const bool overflow = n_win > (uint32_t)WCAP;

    // ---- index: counts per source vertex -----------------------------------------------------
    for (uint32_t i = tid; i < nvert; i += FT) cnt[i] = 0;
    __syncthreads();
    if (!overflow) {
      for (uint32_t i = tid; i < n_win; i += FT) atomicAdd(&cnt[s.ar.vsrc[sm.win[i]] - cbeg], 1u);
    } else {
      // more winners than the shared list: re-stream the log (second pass below scatters)
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
          if (s.ar.key[p] == otk[s.ar.obj[p]]) atomicAdd(&cnt[s.ar.vsrc[p] - cbeg], 1u);
        }
      }
    }
    __syncthreads();
    block_exclusive_scan(cnt, nvert, sm.wsum);
    if (tid == 0) {
      const unsigned long long alloc = (n_win + 3u) & ~3ull;
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
      for (uint32_t i = tid; i < nvert; i += FT) {
        const uint32_t b = cnt[i];
        const uint32_t en = (i + 1 < nvert) ? cnt[i + 1] : n_win;
        s.v_obj[cbeg + i] = make_uint2((uint32_t)(ob0 + b), en - b);
      }
      __syncthreads();
      // ---- scatter the winners' records into R[c] (cursors = per-vertex begin offsets) ---
      if (!overflow) {
        for (uint32_t i = tid; i < n_win; i += FT) {
          const uint32_t p = sm.win[i];
          const uint32_t vs = s.ar.vsrc[p];
          const uint32_t q = (uint32_t)ob0 + atomicAdd(&cnt[vs - cbeg], 1u);
          out.obj[q] = s.ar.obj[p];
          out.key[q] = s.ar.key[p];
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
            if (kk == otk[ob]) {
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
        s.cell_comp[c] = make_uint2((uint32_t)ob0, n_win);
        s.cell_head[c] = NONE;
        s.cell_pending[c] = 0;
        atomicAdd(&st->objects_written, (unsigned long long)n_win);
        atomicAdd(&st->cells_flushed, 1ull);
        atomicAdd(&st->records_flushed, nrec);
      }
    }
    __syncthreads();
    c = c_n;
    head = head_n;
    comp = comp_n;
    c_n = c_nn;
  }
}

template <int HCAP>
void launch_t(const DevGraph& g, const DevState& s, const Arena& out, unsigned long long* out_top,
              uint32_t begin, int sm_count, cudaStream_t st) {
  static int blocks_per_sm = 0;
  const int smem = (int)sizeof(FlushSmem<HCAP>);
  if (blocks_per_sm == 0) {
    cudaFuncSetAttribute(k_flush<HCAP>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    int b = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_flush<HCAP>, FT, smem);
    blocks_per_sm = b > 0 ? b : 1;
  }
  k_flush<HCAP><<<sm_count * blocks_per_sm, FT, smem, st>>>(g, s, out, out_top, begin);
}
}  // namespace

void launch_flush(const DevGraph& g, const DevState& s, const Arena& out,
                  unsigned long long* out_top, uint32_t begin, uint32_t objects_per_cell,
                  int sm_count, cudaStream_t st) {
  (void)objects_per_cell;
  if (g.cs <= 1024) launch_t<1024>(g, s, out, out_top, begin, sm_count, st);
  else launch_t<4096>(g, s, out, out_top, begin, sm_count, st);
}

}  // namespace gg

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
// One CTA cleans one cell at a time (static schedule; the next cells' list entry, head and
// first extent header are loaded one to three cells ahead):
//   gather   the cell's extents (newest first, then its previous cleaned list) into a
//            shared-memory list; they form one logical record sequence tiled across extent
//            boundaries (extents start on 4-record boundaries: every 4-record group is one
//            128-bit load of obj and two of keys).  Each warp streams its own groups with
//            the next group's loads in flight; no barrier inside the stream.
//   match    per record: ot_key[obj] through L1 (a cell touches a few dozen objects, so
//            the lines stay resident), compare; matches are appended to a shared winner list.
//   index    one parallel gather of the winners' payload into shared memory, counts per
//            source vertex, block scan, the bump allocation (issued right after the match,
//            consumed after the scan), v_obj updates (clear the previous list's vertices,
//            set the vertices holding objects now), scatter of R[c] sorted by source vertex.
// A cell with more winners than the shared list falls back to a second streaming pass.
#include <algorithm>

#include "internal.cuh"

#ifdef GG_FLUSH_TIMING
__device__ unsigned long long g_flush_timing[8];
extern "C" int ggrid_debug_flush_timing(unsigned long long* out8) {
  return (int)cudaMemcpyFromSymbol(out8, g_flush_timing, sizeof(g_flush_timing));
}
#define FTS(i) do { if (threadIdx.x == 0) { const long long t_ = clock64(); atomicAdd(&g_flush_timing[i], (unsigned long long)(t_ - ft_prev)); ft_prev = t_; } } while (0)
#else
#define FTS(i) do {} while (0)
#endif

namespace gg {

namespace {
constexpr int FT = 128;        // threads per CTA (8 CTAs per SM)
constexpr int NW = FT / 32;
constexpr int RPT = 4;         // records per lane per group (one 128-bit load of obj)
constexpr int XMAX = 32;       // extents gathered per pass over the chain
constexpr int RANKMAX = 128;   // winners indexed by rank (else per-vertex counters + scan)

template <int HCAP, int WCAP>  // vertex counters, winners staged in shared memory
struct FlushSmem {
  unsigned long long w_key[WCAP];  // staged winners: key, obj, vsrc, off, edge
  uint32_t w_pos[WCAP];
  uint32_t w_obj[WCAP];
  uint32_t w_vs[WCAP];
  uint32_t w_off[WCAP];
  uint32_t w_edge[WCAP];
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

// Gather up to XMAX segments of the cell's log (the previous cleaned list goes last).
// `first` is the header (start, len, next) of chain extent e, prefetched by the caller when
// e is the cell's head.  Thread 0 walks; the list is published in shared memory.
template <class SM>
__device__ void gather_extents(SM& sm, const DevState& s, uint32_t e, uint3 first, uint2 comp) {
  if (threadIdx.x == 0) {
    uint32_t n = 0, pre = 0;
    bool have = true;
    while (e != NONE && n < XMAX) {
      uint32_t st, ln, nxt;
      if (have) {
        st = first.x;
        ln = first.y;
        nxt = first.z;
        have = false;
      } else {
        st = s.x_start[e];
        ln = s.x_len[e];
        nxt = s.x_next[e];
      }
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
    // read-once stream: evict-first, so it does not push the object table out of L1/L2
    r.o = __ldcs(reinterpret_cast<const uint4*>(s.ar.obj + r.pos));
    r.k01 = __ldcs(reinterpret_cast<const ulonglong2*>(s.ar.key + r.pos));
    r.k23 = __ldcs(reinterpret_cast<const ulonglong2*>(s.ar.key + r.pos + 2));
  }
  return r;
}

template <int HCAP, int WCAP>
__global__ void __launch_bounds__(FT, 8) k_flush(DevGraph g, DevState s, Arena out,
                                                 unsigned long long* out_top, uint32_t begin,
                                                 int full_vobj) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  using SM = FlushSmem<HCAP, WCAP>;
  SM& sm = *reinterpret_cast<SM*>(smem_raw);
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const unsigned lt = lanemask_lt();
  DevStatus* st = s.st;
  const uint32_t lend = *((volatile unsigned*)&st->n_flush);
  if (blockIdx.x == 0 && tid == 0) st->flush_end = lend;
  const uint32_t G = gridDim.x;
  const unsigned long long* __restrict__ otk = s.ot_key;
  auto ext_hdr = [&](uint32_t e) {
    return e == NONE ? make_uint3(0, 0, NONE) : make_uint3(s.x_start[e], s.x_len[e], s.x_next[e]);
  };

  // Static schedule (cells li = begin + blockIdx.x + i*G).  Metadata pipeline, consumed one
  // cell later: list entry 3 cells ahead, (head, comp) 2 ahead, first extent header 1 ahead.
  uint32_t li = begin + blockIdx.x;
  uint32_t c0 = li < lend ? s.flush_list[li] : 0;
  uint32_t h0 = li < lend ? s.cell_head[c0] : NONE;
  uint2 p0 = li < lend ? s.cell_comp[c0] : make_uint2(0, 0);
  uint3 x0 = ext_hdr(h0);
  uint32_t c1 = li + G < lend ? s.flush_list[li + G] : 0;
  uint32_t h1 = li + G < lend ? s.cell_head[c1] : NONE;
  uint2 p1 = li + G < lend ? s.cell_comp[c1] : make_uint2(0, 0);
  uint32_t c2 = li + 2 * G < lend ? s.flush_list[li + 2 * G] : 0;
#ifdef GG_FLUSH_TIMING
  long long ft_prev = clock64();
#endif
  for (; li < lend; li += G) {
    FTS(0);
    // issue the pipeline loads for the next cells now (consumed next iteration)
    const uint3 x1 = li + G < lend ? ext_hdr(h1) : make_uint3(0, 0, NONE);
    uint32_t h2 = NONE, c3 = 0;
    uint2 p2 = make_uint2(0, 0);
    if (li + 2 * G < lend) {
      h2 = s.cell_head[c2];
      p2 = s.cell_comp[c2];
    }
    if (li + 3 * G < lend) c3 = s.flush_list[li + 3 * G];

    const uint32_t c = c0, head = h0;
    const uint2 comp = p0;
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
    uint3 first = x0;
    for (;;) {
      __syncthreads();
      gather_extents(sm, s, e, first, comp);
      FTS(1);
      const uint32_t total = sm.xpre[sm.nx];
      if (tid == 0)
        for (uint32_t j = 0; j < sm.nx; ++j) nrec += sm.xl[j];
      // warp w takes groups of 32*RPT records: L = (w + NW*i) * 128 + lane * 4
      int xj = 0;
      uint32_t L = (uint32_t)wid * (32 * RPT) + (uint32_t)lane * RPT;
      Grp cur = load_group(sm, s, L, xj);
      while (__any_sync(0xffffffffu, L < total)) {
        const uint32_t Ln = L + NW * 32 * RPT;
        const Grp nxt = load_group(sm, s, Ln, xj);  // next group's loads in flight
        const uint32_t o[RPT] = {cur.o.x, cur.o.y, cur.o.z, cur.o.w};
        const unsigned long long k[RPT] = {cur.k01.x, cur.k01.y, cur.k23.x, cur.k23.y};
        unsigned long long tg[RPT];
#pragma unroll
        for (int j = 0; j < RPT; ++j)  // all four gathers in flight before the first use
          tg[j] = (uint32_t)j < cur.nv ? __ldg(otk + o[j]) : ~k[j];
#pragma unroll
        for (int j = 0; j < RPT; ++j) {
          const bool hit = tg[j] == k[j];
          const unsigned hm = __ballot_sync(0xffffffffu, hit);
          if (hm) {
            uint32_t base = 0;
            if (lane == __ffs(hm) - 1) base = atomicAdd(&sm.n_win, (unsigned)__popc(hm));
            base = __shfl_sync(0xffffffffu, base, __ffs(hm) - 1);
            const uint32_t w = base + __popc(hm & lt);
            if (hit && w < WCAP) sm.w_pos[w] = cur.pos + j;
          }
        }
        cur = nxt;
        L = Ln;
      }
      __syncthreads();
      if (sm.comp_done) break;
      e = sm.e_next;
      first = ext_hdr(e);
    }
    FTS(2);
    const uint32_t n_win = sm.n_win;
    const bool overflow = n_win > (uint32_t)WCAP;

    // ---- index -------------------------------------------------------------------------------
    // output range: issued now, consumed after staging (the atomic's latency is hidden)
    unsigned long long o0 = 0;
    if (tid == 0) o0 = atomicAdd(out_top, (n_win + 3u) & ~3ull);
    // v_obj entries are self-validating (a vertex's (start, n) counts only if start lies in
    // the cell's current list, and lists only move up the arena between collections), so only
    // the vertices holding objects now are written; garbage collection rewrites every vertex.
    const bool rank_path = !overflow && n_win <= (uint32_t)RANKMAX && !full_vobj;
    if (rank_path) {
      // few winners: one gather round of their payload, then each winner's rank among the
      // winners ordered by (source vertex, index) gives its slot in R[c] — no scan, no counters
      for (uint32_t i = tid; i < n_win; i += FT) {
        const uint32_t p = sm.w_pos[i];
        sm.w_vs[i] = s.ar.vsrc[p];
        sm.w_obj[i] = s.ar.obj[p];
        sm.w_key[i] = s.ar.key[p];
        sm.w_off[i] = s.ar.off[p];
        sm.w_edge[i] = s.ar.edge[p];
      }
      if (tid == 0) {
        sm.out = o0;
        if (o0 + ((n_win + 3u) & ~3ull) > out.cap) {
          sm.fail = 1;
          atomicOr(&st->err, (unsigned)ERR_ARENA);
        }
      }
      __syncthreads();
      FTS(3);
      if (!sm.fail) {
        const uint32_t ob0 = (uint32_t)sm.out;
        for (uint32_t i = tid; i < n_win; i += FT) {
          const uint32_t vi = sm.w_vs[i];
          uint32_t r = 0, cv = 0;
          bool first = true;
          for (uint32_t j = 0; j < n_win; ++j) {
            const uint32_t vj = sm.w_vs[j];
            r += (vj < vi) | ((vj == vi) & (j < i));
            cv += vj == vi;
            first &= !((vj == vi) & (j < i));
          }
          const uint32_t q = ob0 + r;
          out.obj[q] = sm.w_obj[i];
          out.key[q] = sm.w_key[i];
          out.vsrc[q] = vi;
          out.off[q] = sm.w_off[i];
          out.edge[q] = sm.w_edge[i];
          if (first) s.v_obj[vi] = make_uint2(q, cv);
        }
      }
      FTS(4);
    } else {
      for (uint32_t i = tid; i < nvert; i += FT) cnt[i] = 0;
      __syncthreads();
      if (!overflow) {
        for (uint32_t i = tid; i < n_win; i += FT) {
          const uint32_t p = sm.w_pos[i];
          const uint32_t vs = s.ar.vsrc[p];
          sm.w_vs[i] = vs;
          sm.w_obj[i] = s.ar.obj[p];
          sm.w_key[i] = s.ar.key[p];
          sm.w_off[i] = s.ar.off[p];
          sm.w_edge[i] = s.ar.edge[p];
          atomicAdd(&cnt[vs - cbeg], 1u);
        }
      } else {
        // more winners than the staging area: re-stream the log (scattered again below)
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
      FTS(3);
      block_exclusive_scan(cnt, nvert, sm.wsum);
      FTS(4);
      if (tid == 0) {
        sm.out = o0;
        if (o0 + ((n_win + 3u) & ~3ull) > out.cap) {
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
          if (full_vobj || en != b) s.v_obj[cbeg + i] = make_uint2((uint32_t)(ob0 + b), en - b);
        }
        __syncthreads();
        // scatter the winners into R[c] (cursors = per-vertex begin offsets)
        if (!overflow) {
          for (uint32_t i = tid; i < n_win; i += FT) {
            const uint32_t vs = sm.w_vs[i];
            const uint32_t q = (uint32_t)ob0 + atomicAdd(&cnt[vs - cbeg], 1u);
            out.obj[q] = sm.w_obj[i];
            out.key[q] = sm.w_key[i];
            out.vsrc[q] = vs;
            out.off[q] = sm.w_off[i];
            out.edge[q] = sm.w_edge[i];
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
      }
    }
    if (tid == 0 && !sm.fail) {
      s.cell_comp[c] = make_uint2((uint32_t)sm.out, n_win);
      s.cell_head[c] = NONE;
      s.cell_pending[c] = 0;
      atomicAdd(&st->objects_written, (unsigned long long)n_win);
      atomicAdd(&st->cells_flushed, 1ull);
      atomicAdd(&st->records_flushed, nrec);
    }
    __syncthreads();
    FTS(5);
    // rotate the metadata pipeline
    c0 = c1;
    h0 = h1;
    p0 = p1;
    x0 = x1;
    c1 = c2;
    h1 = h2;
    p1 = p2;
    c2 = c3;
  }
}

template <int HCAP, int WCAP>
void launch_t(const DevGraph& g, const DevState& s, const Arena& out, unsigned long long* out_top,
              uint32_t begin, int full_vobj, int sm_count, cudaStream_t st) {
  static int blocks_per_sm = 0;
  const int smem = (int)sizeof(FlushSmem<HCAP, WCAP>);
  if (blocks_per_sm == 0) {
    cudaFuncSetAttribute(k_flush<HCAP, WCAP>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    // ask for no more shared memory than the resident CTAs need: the rest stays L1, which
    // holds the object-table lines the match phase gathers
    const int carve = std::min(100, (8 * (smem + 1024) * 100 + 228 * 1024 - 1) / (228 * 1024));
    cudaFuncSetAttribute(k_flush<HCAP, WCAP>, cudaFuncAttributePreferredSharedMemoryCarveout, carve);
    int b = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_flush<HCAP, WCAP>, FT, smem);
    blocks_per_sm = b > 0 ? b : 1;
  }
  k_flush<HCAP, WCAP><<<sm_count * blocks_per_sm, FT, smem, st>>>(g, s, out, out_top, begin, full_vobj);
}
}  // namespace

void launch_flush(const DevGraph& g, const DevState& s, const Arena& out,
                  unsigned long long* out_top, uint32_t begin, uint32_t objects_per_cell,
                  int full_vobj, int sm_count, cudaStream_t st) {
  // staging sized for ~2x the live objects of an average cell (more winners fall back to a
  // second streaming pass)
  const bool small_h = g.cs <= 1024;
  if (objects_per_cell <= 64) {
    if (small_h) launch_t<1024, 128>(g, s, out, out_top, begin, full_vobj, sm_count, st);
    else launch_t<4096, 128>(g, s, out, out_top, begin, full_vobj, sm_count, st);
  } else if (objects_per_cell <= 256) {
    if (small_h) launch_t<1024, 512>(g, s, out, out_top, begin, full_vobj, sm_count, st);
    else launch_t<4096, 512>(g, s, out, out_top, begin, full_vobj, sm_count, st);
  } else {
    if (small_h) launch_t<1024, 2048>(g, s, out, out_top, begin, full_vobj, sm_count, st);
    else launch_t<4096, 2048>(g, s, out, out_top, begin, full_vobj, sm_count, st);
  }
}

}  // namespace gg

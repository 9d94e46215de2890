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
// Warp-specialised persistent CTAs (static cell schedule), one cell per step, three cells
// in flight per CTA:
//   4 streaming warps   match cell i: the cell's extents (newest first, then its previous
//                       cleaned list) form one logical record sequence tiled across extent
//                       boundaries (extents start on 4-record boundaries: every 4-record
//                       group is one evict-first 128-bit load of obj and two of keys, the next
//                       group's loads in flight); per record ot_key[obj] through L1 (a cell
//                       touches a few dozen objects), compare, append matches to the cell's
//                       shared winner list.
//   1 index warp        meanwhile indexes cell i-1 (one gather round of the winners'
//                       payload, rank by source vertex, bump allocation, scatter of R[c]
//                       sorted by source vertex, v_obj set for the vertices holding objects,
//                       cell marked clean) and gathers the extent list of cell i+2.
// One CTA barrier per step.  Cells with more winners than the rank path handles, or GC's
// full v_obj rewrite, take a counter + warp-scan path; the positions of winners beyond the
// shared-memory staging (WCAP) spill to a per-CTA global area, and only a cell that overflows
// that too is re-streamed by the index warp.
#include <algorithm>

#include "internal.cuh"

namespace gg {

namespace {
#ifndef GG_SW
#define GG_SW 4
#endif
constexpr int SW = GG_SW;           // streaming warps
constexpr int FT = (SW + 1) * 32;   // + one index warp
constexpr int RPT = 4;              // records per lane per group (one 128-bit load of obj)
constexpr uint32_t STRIDE = SW * 32 * RPT;
constexpr int XMAX = 32;            // extents gathered per pass over the chain
constexpr int RANKMAX = 128;        // winners indexed by rank (else counters + scan)
constexpr int NBUF = 3;             // cells in flight: gathering, streaming, indexing

template <int WCAP>
struct CellBuf {
  uint32_t xs[XMAX];
  uint32_t xl[XMAX];
  uint32_t xpre[XMAX + 1];
  uint32_t nx, e_next, comp_done;
  uint32_t c, head, has;  // cell id, chain head, this buffer holds a cell
  uint2 comp;             // previous cleaned list
  unsigned long long nrec;
  unsigned long long nexp;  // records of extents dropped by t_delta expiry
  uint32_t n_win;
  uint32_t spill_cap;     // this buffer's global spill area (winners beyond WCAP)
  uint32_t* spill;
  uint32_t w_pos[WCAP];   // arena positions of the matched records
};

template <int HCAP, int WCAP>
struct FlushSmem {
  CellBuf<WCAP> b[NBUF];
  // index warp only
  unsigned long long w_key[WCAP];
  uint32_t w_obj[WCAP];
  uint32_t w_vs[WCAP];
  uint32_t w_off[WCAP];
  uint32_t w_edge[WCAP];
  uint32_t hist[HCAP];
};

__device__ __forceinline__ void stream_bar() { asm volatile("bar.sync 1, %0;" ::"n"(SW * 32)); }

// Walk up to XMAX extents of a chain starting at e into buffer bf; the cleaned list `comp`
// goes last.  One lane.
// Extents whose newest message is older than t_cut are expired: skipped unread (the paper's
// bucket discard at cleaning time, P@20631-21157, reading R21).
template <class B>
__device__ void walk_extents(B& bf, const DevState& s, uint32_t e, uint2 comp, uint32_t t_cut) {
  uint32_t n = 0, pre = 0;
  unsigned long long nrec = 0, nexp = 0;
  while (is_extent(e) && n < XMAX) {
    const uint32_t st = s.x_start[e], ln = s.x_len[e], nxt = s.x_next[e];
    if (t_cut && s.x_tmax[e] < t_cut) {
      nexp += ln;
      e = nxt;
      continue;
    }
    bf.xs[n] = st;
    bf.xl[n] = ln;
    bf.xpre[n] = pre;
    pre += (ln + 3u) & ~3u;
    nrec += ln;
    ++n;
    e = nxt;
  }
  bf.comp_done = 0;
  if (!is_extent(e) && n < XMAX) {
    if (comp.y) {
      bf.xs[n] = comp.x;
      bf.xl[n] = comp.y;
      bf.xpre[n] = pre;
      pre += (comp.y + 3u) & ~3u;
      nrec += comp.y;
      ++n;
    }
    bf.comp_done = 1;
  }
  bf.xpre[n] = pre;
  bf.nx = n;
  bf.e_next = e;
  bf.nrec += nrec;
  bf.nexp += nexp;
}

struct Grp {
  uint4 o;
  ulonglong2 k01, k23;
  uint32_t pos;  // arena position of the group's first record
  uint32_t nv;   // valid records in the group (0..4)
};

// The 4-record group at logical offset L (a multiple of 4).  j is the lane's extent cursor
// (L only grows along a lane's stream, so j only advances).
template <class B>
__device__ __forceinline__ Grp load_group(const B& bf, const DevState& s, uint32_t L, int& j) {
  Grp r;
  r.nv = 0;
  r.pos = 0;
  if (L >= bf.xpre[bf.nx]) return r;
  while (j + 1 < (int)bf.nx && bf.xpre[j + 1] <= L) ++j;
  const uint32_t off = L - bf.xpre[j];
  r.pos = bf.xs[j] + off;
  const uint32_t len = bf.xl[j];
  r.nv = off >= len ? 0 : min(4u, len - off);
  if (r.nv) {
    // read-once stream: evict-first, so it does not push the object table out of L1/L2
    r.o = __ldcs(reinterpret_cast<const uint4*>(s.ar.obj + r.pos));
    r.k01 = __ldcs(reinterpret_cast<const ulonglong2*>(s.ar.key + r.pos));
    r.k23 = __ldcs(reinterpret_cast<const ulonglong2*>(s.ar.key + r.pos + 2));
  }
  return r;
}

// streaming warps: match the gathered extent list of buffer bf
template <int WCAP, class B>
__device__ __forceinline__ void stream_list(B& bf, const DevState& s, int sw, int lane, unsigned lt) {
  const unsigned long long* __restrict__ otk = s.ot_key;
  const uint32_t total = bf.xpre[bf.nx];
  int xj = 0;
  uint32_t L = (uint32_t)sw * (32 * RPT) + (uint32_t)lane * RPT;
  Grp cur = load_group(bf, s, L, xj);
  while (__any_sync(0xffffffffu, L < total)) {
    const uint32_t Ln = L + STRIDE;
    const Grp nxt = load_group(bf, s, Ln, xj);  // next group's loads in flight
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
        if (lane == __ffs(hm) - 1) base = atomicAdd(&bf.n_win, (unsigned)__popc(hm));
        base = __shfl_sync(0xffffffffu, base, __ffs(hm) - 1);
        const uint32_t w = base + __popc(hm & lt);
        if (hit) {
          if (w < (uint32_t)WCAP) bf.w_pos[w] = cur.pos + j;
          else if (w - (uint32_t)WCAP < bf.spill_cap) bf.spill[w - WCAP] = cur.pos + j;  // (rare)
        }
      }
    }
    cur = nxt;
    L = Ln;
  }
}

// index warp: exclusive scan of a[0..n) (smem or global); returns the total
__device__ uint32_t warp_exclusive_scan(uint32_t* a, uint32_t n, int lane) {
  uint32_t carry = 0;
  for (uint32_t b0 = 0; b0 < n; b0 += 32) {
    const uint32_t i = b0 + lane;
    const uint32_t v = i < n ? a[i] : 0;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (i < n) a[i] = carry + x - v;
    carry += __shfl_sync(0xffffffffu, x, 31);
  }
  return carry;
}

// index warp: build R[c] for the cell of buffer bf (whose winners are known)
template <int HCAP, int WCAP, class SM, class B>
__device__ void index_cell(SM& sm, B& bf, const DevGraph& g, const DevState& s, const Arena& out,
                           unsigned long long* out_top, int full_vobj, int lane,
                           const uint32_t* __restrict__ spill, uint32_t spill_cap, uint32_t t_cut) {
  const unsigned long long* __restrict__ otk = s.ot_key;
  const uint32_t c = bf.c, head = bf.head;
  const uint2 comp = bf.comp;
  const uint32_t n_win = bf.n_win;
  // winners: staged in shared memory (<= WCAP), positions spilled to this buffer's global
  // spill area (<= WCAP + spill_cap), else the cell's log is re-streamed (overflow)
  const bool spilled = n_win > (uint32_t)WCAP && n_win - (uint32_t)WCAP <= spill_cap;
  const bool overflow = n_win > (uint32_t)WCAP && !spilled;
  const bool staged = !spilled && !overflow;
  auto wpos = [&](uint32_t i) { return i < (uint32_t)WCAP ? bf.w_pos[i] : spill[i - WCAP]; };
  const uint32_t cbeg = c * g.cs;
  const uint32_t nvert = min(g.cs, g.V - cbeg);
  unsigned long long o0 = 0;
  if (lane == 0) o0 = atomicAdd(out_top, (n_win + 3u) & ~3ull);  // consumed after staging
  if (staged) {
    for (uint32_t i = lane; i < n_win; i += 32) {  // one gather round of the payload
      const uint32_t p = bf.w_pos[i];
      sm.w_vs[i] = s.ar.vsrc[p];
      sm.w_obj[i] = s.ar.obj[p];
      sm.w_key[i] = s.ar.key[p];
      sm.w_off[i] = s.ar.off[p];
      sm.w_edge[i] = s.ar.edge[p];
    }
  }
  o0 = __shfl_sync(0xffffffffu, o0, 0);
  const bool fail = o0 + ((n_win + 3u) & ~3ull) > out.cap;
  __syncwarp();
  if (fail) {
    if (lane == 0) atomicOr(&s.st->err, (unsigned)ERR_ARENA);
    return;  // the cell stays dirty
  }
  const uint32_t ob0 = (uint32_t)o0;
  // (GG_VHAS) the cell's "may hold objects" bits: cleared, then set below for the new list
  // (boundary words shared with a neighbouring cell: masked atomics)
  for (uint32_t wd = (cbeg >> 5) + lane; GG_VHAS && wd <= ((cbeg + nvert - 1) >> 5); wd += 32) {
    const uint32_t lo = max(cbeg, wd << 5), hi = min(cbeg + nvert, (wd << 5) + 32);
    const uint32_t span = hi - lo;
    const uint32_t mask = (span == 32 ? 0xFFFFFFFFu : ((1u << span) - 1u)) << (lo & 31);
    atomicAnd(&s.vhas[wd], ~mask);
  }
  __syncwarp();
  // v_obj entries are self-validating (vobj_valid): only vertices holding objects now are
  // written; garbage collection (full_vobj) rewrites every vertex of the cell.
  if (staged && n_win <= (uint32_t)RANKMAX && !full_vobj) {
    // slot of a winner = its rank among the winners ordered by (source vertex, index)
    for (uint32_t i = lane; i < n_win; i += 32) {
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
      s.listed_cell[sm.w_obj[i]] = c;
      out.obj[q] = sm.w_obj[i];
      out.key[q] = sm.w_key[i];
      out.vsrc[q] = vi;
      out.off[q] = sm.w_off[i];
      out.edge[q] = sm.w_edge[i];
      if (first) {
        s.v_obj[vi] = make_uint2(q, cv);
        if (GG_VHAS) atomicOr(&s.vhas[vi >> 5], 1u << (vi & 31));
      }
    }
  } else {
    uint32_t* cnt = (nvert <= (uint32_t)HCAP) ? sm.hist : (s.vcnt + cbeg);
    for (uint32_t i = lane; i < nvert; i += 32) cnt[i] = 0;
    __syncwarp();
    // records of the cell's log in chain order (only for the > WCAP fallback)
    auto for_each_record = [&](auto&& fn) {
      uint32_t e2 = head;
      bool last = false;
      while (!last) {
        uint32_t sst, sln;
        if (is_extent(e2)) {
          sst = s.x_start[e2];
          sln = (t_cut && s.x_tmax[e2] < t_cut) ? 0u : s.x_len[e2];
          e2 = s.x_next[e2];
        } else {
          sst = comp.x;
          sln = comp.y;
          last = true;
        }
        for (uint32_t r = lane; r < sln; r += 32) fn(sst + r);
      }
    };
    if (staged) {
      for (uint32_t i = lane; i < n_win; i += 32) atomicAdd(&cnt[sm.w_vs[i] - cbeg], 1u);
    } else if (spilled) {
      constexpr int U = 4;  // four winners per lane in flight
      for (uint32_t i0 = lane; i0 < n_win; i0 += 32 * U) {
        uint32_t p[U], vs[U];
#pragma unroll
        for (int u = 0; u < U; ++u) p[u] = i0 + u * 32 < n_win ? wpos(i0 + u * 32) : 0;
#pragma unroll
        for (int u = 0; u < U; ++u) vs[u] = i0 + u * 32 < n_win ? s.ar.vsrc[p[u]] : 0;
#pragma unroll
        for (int u = 0; u < U; ++u)
          if (i0 + u * 32 < n_win) atomicAdd(&cnt[vs[u] - cbeg], 1u);
      }
    } else {
      for_each_record([&](uint32_t p) {
        if (s.ar.key[p] == otk[s.ar.obj[p]]) atomicAdd(&cnt[s.ar.vsrc[p] - cbeg], 1u);
      });
    }
    __syncwarp();
    warp_exclusive_scan(cnt, nvert, lane);
    __syncwarp();
    for (uint32_t i = lane; i < nvert; i += 32) {
      const uint32_t b = cnt[i];
      const uint32_t en = (i + 1 < nvert) ? cnt[i + 1] : n_win;
      if (full_vobj || en != b) s.v_obj[cbeg + i] = make_uint2(ob0 + b, en - b);
      if (GG_VHAS && en != b) atomicOr(&s.vhas[(cbeg + i) >> 5], 1u << ((cbeg + i) & 31));
    }
    __syncwarp();
    if (spilled) {
      constexpr int U = 2;  // (the kernel's register count is set by its widest path)
      for (uint32_t i0 = lane; i0 < n_win; i0 += 32 * U) {
        uint32_t p[U], ob[U], vs[U], of[U], ed[U];
        unsigned long long kk[U];
#pragma unroll
        for (int u = 0; u < U; ++u) p[u] = i0 + u * 32 < n_win ? wpos(i0 + u * 32) : 0;
#pragma unroll
        for (int u = 0; u < U; ++u) {
          ob[u] = s.ar.obj[p[u]];
          kk[u] = s.ar.key[p[u]];
          vs[u] = s.ar.vsrc[p[u]];
          of[u] = s.ar.off[p[u]];
          ed[u] = s.ar.edge[p[u]];
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          if (i0 + u * 32 >= n_win) continue;
          const uint32_t q = ob0 + atomicAdd(&cnt[vs[u] - cbeg], 1u);
          s.listed_cell[ob[u]] = c;
          out.obj[q] = ob[u];
          out.key[q] = kk[u];
          out.vsrc[q] = vs[u];
          out.off[q] = of[u];
          out.edge[q] = ed[u];
        }
      }
    } else if (staged) {
      for (uint32_t i = lane; i < n_win; i += 32) {
        const uint32_t vs = sm.w_vs[i];
        const uint32_t q = ob0 + atomicAdd(&cnt[vs - cbeg], 1u);
        s.listed_cell[sm.w_obj[i]] = c;
        out.obj[q] = sm.w_obj[i];
        out.key[q] = sm.w_key[i];
        out.vsrc[q] = vs;
        out.off[q] = sm.w_off[i];
        out.edge[q] = sm.w_edge[i];
      }
    } else {
      for_each_record([&](uint32_t p) {
        const uint32_t ob = s.ar.obj[p];
        const unsigned long long kk = s.ar.key[p];
        if (kk == otk[ob]) {
          const uint32_t vs = s.ar.vsrc[p];
          const uint32_t q = ob0 + atomicAdd(&cnt[vs - cbeg], 1u);
          s.listed_cell[ob] = c;
          out.obj[q] = ob;
          out.key[q] = kk;
          out.vsrc[q] = vs;
          out.off[q] = s.ar.off[p];
          out.edge[q] = s.ar.edge[p];
        }
      });
    }
  }
  if (lane == 0) {
    s.cell_comp[c] = make_uint2(ob0, n_win);
    s.cell_head[c] = NONE;
    s.cell_pending[c] = 0;
    atomicAdd(&s.st->objects_written, (unsigned long long)n_win);
    atomicAdd(&s.st->cells_flushed, 1ull);
    atomicAdd(&s.st->records_flushed, bf.nrec);
    if (bf.nexp) atomicAdd(&s.st->records_expired, bf.nexp);
  }
}

template <int HCAP, int WCAP>
// 7 resident CTAs per SM (56 registers, a few spills): more 128-bit streams in flight than
// ptxas's own 64-register choice (6 CTAs): C3 flush 52.5% -> 56% of measured HBM bandwidth
// (8 CTAs: 54.4%; an explicit 1 lets ptxas take 96 registers: 42%)
#ifndef GG_FLUSH_MINB
#define GG_FLUSH_MINB 7
#endif
__global__ void __launch_bounds__(FT, GG_FLUSH_MINB) k_flush(DevGraph g, DevState s, Arena out,
                                              unsigned long long* out_top, uint32_t begin,
                                              int full_vobj, uint32_t* spill, uint32_t spill_cap,
                                              uint32_t t_cut) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  using SM = FlushSmem<HCAP, WCAP>;
  SM& sm = *reinterpret_cast<SM*>(smem_raw);
  pdl_wait();   // (a programmatic dependent of the seed / status reset)
  pdl_allow();  // the expansion may launch now (it waits for this grid before reading)
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const unsigned lt = lanemask_lt();
  // begin == OVF_PASS: the cells k_flush_warp left (s.ovf_list), not the request list
  const bool ovf_pass = begin == OVF_PASS;
  const uint32_t* __restrict__ flist = ovf_pass ? s.ovf_list : s.flush_list;
  const uint32_t lend = *((volatile unsigned*)(ovf_pass ? &s.st->n_ovf : &s.st->n_flush));
  if (ovf_pass) begin = 0;
  else if (blockIdx.x == 0 && tid == 0) s.st->flush_end = lend;
  const uint32_t G = gridDim.x;
  const uint32_t first_li = begin + blockIdx.x;
  const uint32_t n_mine = first_li < lend ? (lend - first_li + G - 1) / G : 0;
  const bool is_index = wid == SW;
  // this CTA's spill area of buffer k % NBUF
  auto spill_of = [&](uint32_t k) {
    return spill + ((size_t)blockIdx.x * NBUF + k % NBUF) * spill_cap;
  };

  // index-warp lane 0 gathers cells ahead of the stream; the next cell's list entry, chain
  // head and cleaned list are loaded one gather ahead
  uint32_t pc = 0, ph = NONE;
  uint2 pcomp = make_uint2(0, 0);
  auto gather = [&](uint32_t k) {  // cell k of this CTA into buffer k % NBUF
    auto& bf = sm.b[k % NBUF];
    bf.n_win = 0;
    bf.nrec = 0;
    bf.nexp = 0;
    bf.spill = spill_of(k);
    bf.spill_cap = spill_cap;
    bf.has = k < n_mine;
    if (!bf.has) {
      bf.nx = 0;
      bf.xpre[0] = 0;
      bf.comp_done = 1;
      return;
    }
    const uint32_t c = pc, head = ph;
    const uint2 comp = pcomp;
    if (k + 1 < n_mine) {
      pc = flist[first_li + (k + 1) * G];
      ph = s.cell_head[pc];
      pcomp = s.cell_comp[pc];
    }
    bf.c = c;
    bf.head = head;
    bf.comp = comp;
    walk_extents(bf, s, head, comp, t_cut);
  };

  if (is_index && lane == 0 && n_mine) {
    pc = flist[first_li];
    ph = s.cell_head[pc];
    pcomp = s.cell_comp[pc];
    gather(0);
    gather(1);
  }
  __syncthreads();
  // step k: streaming warps match cell k; the index warp indexes cell k-1 and gathers k+2
  for (uint32_t k = 0; k <= n_mine; ++k) {
    if (!is_index) {
      auto& bf = sm.b[k % NBUF];
      if (k < n_mine) {
        for (;;) {
          stream_list<WCAP>(bf, s, wid, lane, lt);
          if (bf.comp_done) break;
          // chains longer than XMAX extents: the streaming warps gather the next part
          stream_bar();
          if (tid == 0) walk_extents(bf, s, bf.e_next, bf.comp, t_cut);
          stream_bar();
        }
      }
    } else {
      if (k >= 1)
        index_cell<HCAP, WCAP>(sm, sm.b[(k - 1) % NBUF], g, s, out, out_top, full_vobj, lane,
                               spill_of(k - 1), spill_cap, t_cut);
      if (lane == 0) gather(k + 2);
      __syncwarp();
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------------------------------------
// Warp-per-cell variant for short logs (a step's few dozen new records per cell, C3: ~43 new + ~43
// listed): the CTA-per-cell pipelines above run a CTA's cells one after another through one index
// warp, so a flush of every cell costs ~23 cells x the index warp's dependent chain per CTA.
// Here each warp takes whole cells from a dynamic counter and runs every phase of one cell
// itself -- chain walk, match (records in flight 4 per lane), winner payload gather, rank by
// source vertex, scatter of R[c] -- with no CTA barrier: ~8k cells are in flight on the GPU at
// once instead of ~1k.  Same arithmetic as index_cell (the staged, rank path).  A cell with more
// than XW extents or more than WW winners is left to the CTA kernel: queued on ovf_list, which
// the launcher hands to k_flush right after.
constexpr int XW = 32;    // extents (including the cleaned list) per cell
constexpr int WW = 128;   // winners per cell
constexpr int FW = 8;     // warps per CTA
struct WarpFlushSmem {
  uint32_t xs[XW], xp[XW + 1];
  uint32_t w_pos[WW], w_obj[WW], w_vs[WW], w_off[WW], w_edge[WW];
  unsigned long long w_key[WW];
  unsigned long long srt[WW];  // (source vertex << 32 | winner index), sorted: R[c]'s order
};

__global__ void __launch_bounds__(FW * 32, 5) k_flush_warp(DevGraph g, DevState s, Arena out,
                                                          unsigned long long* out_top, uint32_t begin,
                                                          uint32_t* ovf_list, uint32_t t_cut) {
  __shared__ WarpFlushSmem wsm[FW];
  pdl_wait();   // (a programmatic dependent of the seed / status reset)
  pdl_allow();  // the overflow pass / expansion may launch now (they wait for this grid)
  const int lane = threadIdx.x & 31;
  WarpFlushSmem& m = wsm[threadIdx.x >> 5];
  const unsigned lt = lanemask_lt();
  const unsigned long long* __restrict__ otk = s.ot_key;
  const uint32_t lend = *((volatile unsigned*)&s.st->n_flush);
  if (blockIdx.x == 0 && threadIdx.x == 0) s.st->flush_end = lend;
  unsigned long long n_written = 0, n_cells = 0, n_rec = 0, n_exp = 0;
  // static schedule: warp w takes list entries begin + w, + W, ... (a shared work counter is one
  // contended address: measured 45% of this kernel's stall samples)
  const uint32_t W = gridDim.x * FW;
  for (uint32_t li = begin + blockIdx.x * FW + (threadIdx.x >> 5); li < lend; li += W) {
    const uint32_t c = s.flush_list[li];
    const uint32_t head = s.cell_head[c];
    const uint2 comp = s.cell_comp[c];
    // ---- the cell's record sequence: its extents newest first (unexpired), then its cleaned list
    uint32_t nx = 0, tot = 0, nexp = 0;
    bool ovf = false;
    if (lane == 0) {
      uint32_t e = head;
      while (is_extent(e)) {
        const uint32_t st = s.x_start[e], ln = s.x_len[e], nxt = s.x_next[e];
        if (t_cut && s.x_tmax[e] < t_cut) {
          nexp += ln;
        } else if (nx + 1 >= (uint32_t)XW) {
          ovf = true;
          break;
        } else if (ln) {
          m.xs[nx] = st;
          m.xp[nx] = tot;
          tot += ln;
          ++nx;
        }
        e = nxt;
      }
      if (comp.y) {
        m.xs[nx] = comp.x;
        m.xp[nx] = tot;
        tot += comp.y;
        ++nx;
      }
      m.xp[nx] = tot;
    }
    nx = __shfl_sync(0xffffffffu, nx, 0);
    tot = __shfl_sync(0xffffffffu, tot, 0);
    ovf = __shfl_sync(0xffffffffu, ovf, 0);
    __syncwarp();
    // ---- match: the record whose key equals ot_key[obj] is its object's latest (R8)
    uint32_t n_win = 0;
    for (uint32_t b0 = 0; b0 < tot && !ovf; b0 += 128) {
      uint32_t p[4], o[4];
      unsigned long long k[4], tg[4];
      int xj = 0;
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const uint32_t L = b0 + u * 32 + lane;
        p[u] = NONE;
        if (L < tot) {
          while (m.xp[xj + 1] <= L) ++xj;
          p[u] = m.xs[xj] + (L - m.xp[xj]);
        }
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        o[u] = p[u] != NONE ? __ldcs(s.ar.obj + p[u]) : 0u;
        k[u] = p[u] != NONE ? __ldcs(s.ar.key + p[u]) : 0ull;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) tg[u] = p[u] != NONE ? __ldg(otk + o[u]) : ~k[u];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const bool hit = tg[u] == k[u];
        const unsigned hm = __ballot_sync(0xffffffffu, hit);
        const uint32_t w = n_win + __popc(hm & lt);
        if (hit && w < (uint32_t)WW) {
          m.w_pos[w] = p[u];
          m.w_obj[w] = o[u];
          m.w_key[w] = k[u];
        }
        n_win += __popc(hm);
      }
      if (n_win > (uint32_t)WW) ovf = true;
    }
    if (ovf) {  // the CTA kernel's spill / re-stream paths take it (right after this launch)
      if (lane == 0) ovf_list[atomicAdd(&s.st->n_ovf, 1u)] = c;
      continue;
    }
    __syncwarp();
    // ---- R[c]: payload gather, then each winner's slot = its rank by (source vertex, index)
    unsigned long long o0 = 0;
    if (lane == 0) o0 = atomicAdd(out_top, (n_win + 3u) & ~3ull);
    for (uint32_t i = lane; i < n_win; i += 32) {
      const uint32_t pp = m.w_pos[i];
      m.w_vs[i] = s.ar.vsrc[pp];
      m.w_off[i] = s.ar.off[pp];
      m.w_edge[i] = s.ar.edge[pp];
    }
    o0 = __shfl_sync(0xffffffffu, o0, 0);
    __syncwarp();
    if (o0 + ((n_win + 3u) & ~3ull) > out.cap) {
      if (lane == 0) atomicOr(&s.st->err, (unsigned)ERR_ARENA);
      continue;  // the cell stays dirty
    }
    const uint32_t cbeg = c * g.cs;
    if (GG_VHAS) {  // the cell's "may hold objects" bits: cleared, then set for the new list
      const uint32_t nvert = min(g.cs, g.V - cbeg);
      for (uint32_t wd = (cbeg >> 5) + lane; wd <= ((cbeg + nvert - 1) >> 5); wd += 32) {
        const uint32_t lo = max(cbeg, wd << 5), hi = min(cbeg + nvert, (wd << 5) + 32);
        const uint32_t span = hi - lo;
        const uint32_t mask = (span == 32 ? 0xFFFFFFFFu : ((1u << span) - 1u)) << (lo & 31);
        atomicAnd(&s.vhas[wd], ~mask);
      }
      __syncwarp();
    }
    // R[c] sorted by (source vertex, winner index): a warp bitonic sort of the packed pairs --
    // in registers (element j * 32 + lane in v[j], shuffles for strides below 32) on 32-bit keys
    // ((vertex - cell base) << 7 | index) when the cell size allows, else in shared memory
    uint32_t n2 = 1;
    while (n2 < n_win) n2 <<= 1;
    if (g.cs <= (1u << 25)) {
      uint32_t v[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t i = j * 32 + lane;
        v[j] = i < n_win ? ((m.w_vs[i] - cbeg) << 7 | i) : 0xFFFFFFFFu;
      }
      const uint32_t E = n2 > 32 ? n2 / 32 : 1;  // registers in use (n2 <= WW = 128)
      for (uint32_t size = 2; size <= n2; size <<= 1) {
        for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
          if (stride >= 32) {  // partner in this lane: register j ^ (stride / 32)
            const uint32_t jj = stride >> 5;
#pragma unroll
            for (uint32_t j = 0; j < 4; ++j) {
              if (j >= E || (j & jj)) continue;
              const bool asc = ((j * 32 + lane) & size) == 0;
              const uint32_t a = v[j], b = v[j | jj];
              if ((a > b) == asc) {
                v[j] = b;
                v[j | jj] = a;
              }
            }
          } else {  // partner in lane ^ stride, same register
#pragma unroll
            for (uint32_t j = 0; j < 4; ++j) {
              if (j >= E) continue;
              const uint32_t o = __shfl_xor_sync(0xffffffffu, v[j], stride);
              const bool asc = ((j * 32 + lane) & size) == 0;
              const bool lower = (lane & stride) == 0;
              v[j] = (lower == asc) ? min(v[j], o) : max(v[j], o);
            }
          }
        }
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t i = j * 32 + lane;
        if (i < n_win) m.srt[i] = ((unsigned long long)((v[j] >> 7) + cbeg) << 32) | (v[j] & 127u);
      }
      __syncwarp();
    } else {
      for (uint32_t i = lane; i < n2; i += 32)
        m.srt[i] = i < n_win ? ((unsigned long long)m.w_vs[i] << 32 | i) : EMPTY64;
      __syncwarp();
      for (uint32_t size = 2; size <= n2; size <<= 1) {
        for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
          for (uint32_t i = lane; i < n2 / 2; i += 32) {
            const uint32_t lo = 2 * i - (i & (stride - 1));
            const uint32_t hi = lo + stride;
            const bool asc = (lo & size) == 0;
            const unsigned long long x = m.srt[lo], y = m.srt[hi];
            if ((x > y) == asc) {
              m.srt[lo] = y;
              m.srt[hi] = x;
            }
          }
          __syncwarp();
        }
      }
    }
    for (uint32_t r = lane; r < n_win; r += 32) {
      const unsigned long long e = m.srt[r];
      const uint32_t i = (uint32_t)e, vi = (uint32_t)(e >> 32);
      const uint32_t q = (uint32_t)o0 + r;
      s.listed_cell[m.w_obj[i]] = c;
      out.obj[q] = m.w_obj[i];
      out.key[q] = m.w_key[i];
      out.vsrc[q] = vi;
      out.off[q] = m.w_off[i];
      out.edge[q] = m.w_edge[i];
      if (r == 0 || (uint32_t)(m.srt[r - 1] >> 32) != vi) {  // the vertex's first object
        uint32_t cv = 1;
        while (r + cv < n_win && (uint32_t)(m.srt[r + cv] >> 32) == vi) ++cv;
        s.v_obj[vi] = make_uint2(q, cv);
        if (GG_VHAS) atomicOr(&s.vhas[vi >> 5], 1u << (vi & 31));
      }
    }
    if (lane == 0) {
      s.cell_comp[c] = make_uint2((uint32_t)o0, n_win);
      s.cell_head[c] = NONE;
      s.cell_pending[c] = 0;
    }
    n_written += n_win;
    n_cells += 1;
    n_rec += tot;
    n_exp += nexp;
    __syncwarp();  // (the staging is rewritten by the next cell)
  }
  if (lane == 0 && n_cells) {
    atomicAdd(&s.st->objects_written, n_written);
    atomicAdd(&s.st->cells_flushed, n_cells);
    atomicAdd(&s.st->records_flushed, n_rec);
    if (n_exp) atomicAdd(&s.st->records_expired, n_exp);
  }
}

// ---------------------------------------------------------------------------------------------
// Bulk-copy (TMA engine) variant of the flush: the record stream of a CTA's cells never drains at
// a cell boundary.  Warp roles (6 warps):
//   producer (warp 0, one lane)  walks each cell's extent chain (+ its previous cleaned list) and
//                                issues cp.async.bulk copies of CHUNK-record pieces of the obj and
//                                key arrays into a ring of TS shared-memory stages, each stage's
//                                landing signalled on its "full" mbarrier (transaction bytes);
//   4 match warps                take the stages round-robin: ot_key[obj] gather (L1/L2), compare,
//                                ballot-append the matching positions to the cell's winner list,
//                                release the stage ("empty" mbarrier); the warp finishing a cell's
//                                last piece queues the cell for indexing;
//   index warp (warp 5)          builds R[c] of each matched cell (index_cell above) and frees its
//                                slot for the producer.
// Up to TSLOT cells are in flight per CTA.  The per-cell arithmetic is the one above.
#ifndef GG_TCHUNK
#define GG_TCHUNK 256
#endif
// 4 stages x 2 match warps: a small ring and 128 threads per CTA = 8 CTAs (cell pipelines) per SM
// at 64 registers; C3 full flush 0.223 ms (8 x 4) -> 0.214-0.217 ms, 58.7% of measured HBM.
// Larger rings or more match warps cost CTAs per SM and lose; register caps spill and lose
// (profiles/flush_tma_*_r2*.log)
#ifndef GG_TS
#define GG_TS 4
#endif
#ifndef GG_TMW
#define GG_TMW 2
#endif
constexpr int TCHUNK = GG_TCHUNK;  // records per stage (8 per match-warp lane)
constexpr int TS = GG_TS;          // stages
constexpr int TSLOT = 4;           // cells in flight
constexpr int TMW = GG_TMW;        // match warps
// each stage must always be consumed by the same match warp (stage s: sequence numbers s, s + TS,
// ... go to warp s % TMW): a warp waiting on a phase two ahead of its stage's barrier would read
// the parity of an older phase as complete
static_assert(TS % TMW == 0, "stages must be a multiple of the match warps");
constexpr int TFT = (TMW + 2) * 32;

template <int WCAP>
struct TSlot {
  uint32_t c, head, has;
  uint2 comp;
  unsigned long long nrec, nexp;
  uint32_t n_win;
  unsigned long long state;  // (pieces of the cell << 32) + pieces matched: complete when equal
  uint32_t spill_cap;
  uint32_t* spill;
  uint32_t w_pos[WCAP];
};

template <int HCAP, int WCAP>
struct TFlushSmem {
  uint32_t obj[TS][TCHUNK];
  unsigned long long key[TS][TCHUNK];
  unsigned long long full[TS], empty[TS];
  uint32_t st_slot[TS], st_n[TS], st_pos[TS];
  TSlot<WCAP> slot[TSLOT];
  uint32_t slot_gen[TSLOT];  // cells indexed per slot (the producer reuses a slot when caught up)
  uint32_t rq[TSLOT];        // matched cells for the index warp: entry i = slot | (i / TSLOT) << 4
  uint32_t rq_n;             // entries pushed
  // index warp only (index_cell)
  unsigned long long w_key[WCAP];
  uint32_t w_obj[WCAP];
  uint32_t w_vs[WCAP];
  uint32_t w_off[WCAP];
  uint32_t w_edge[WCAP];
  uint32_t hist[HCAP];
};

#ifndef GG_MBAR_SUSPEND_NS
#define GG_MBAR_SUSPEND_NS 1000000
#endif
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
// (a suspend-time hint: the waiting warp sleeps until the phase completes instead of spinning
// through try_wait, which took ~16% of the kernel's issue slots at C3)
__device__ __forceinline__ void mbar_wait(unsigned long long* b, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n"
      "W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n @!p bra W_%=;\n}" ::"r"(smem_u32(b)),
      "r"(parity), "r"(GG_MBAR_SUSPEND_NS)
      : "memory");
}
// global -> shared bulk copy (TMA engine; 16-byte aligned, multiple of 16 bytes), evict-first in
// L2 (the log is read once)
__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, unsigned long long* bar,
                                          unsigned long long policy) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
      : "memory");
}

// queue a matched cell for the index warp (at most TSLOT entries are pending: one per slot)
__device__ __forceinline__ void rq_push(uint32_t* rq_n, uint32_t* rq, uint32_t b) {
  __threadfence_block();  // (the cell's winners before its entry)
  const uint32_t i = atomicAdd(rq_n, 1u);
  ((volatile uint32_t*)rq)[i % TSLOT] = b | ((i / TSLOT) << 4);
}

template <int HCAP, int WCAP>
// (an explicit min-blocks bound -- even 1 -- changes ptxas's register choice: 72 registers, 4 CTAs
// per SM, 0.233 ms at C3 vs 56 registers, 5 CTAs, 0.223 ms without one; r2 profiling pass)
#ifdef GG_TMA_MINB
#define TMA_BOUNDS __launch_bounds__(TFT, GG_TMA_MINB)
#else
#define TMA_BOUNDS __launch_bounds__(TFT)
#endif
__global__ void TMA_BOUNDS k_flush_tma(DevGraph g, DevState s, Arena out, unsigned long long* out_top,
                                                   uint32_t begin, int full_vobj, uint32_t* spill, uint32_t spill_cap,
                                                   uint32_t t_cut) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  using SM = TFlushSmem<HCAP, WCAP>;
  SM& sm = *reinterpret_cast<SM*>(smem_raw);
  pdl_wait();
  pdl_allow();
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const unsigned lt = lanemask_lt();
  const uint32_t lend = *((volatile unsigned*)&s.st->n_flush);
  if (blockIdx.x == 0 && tid == 0) s.st->flush_end = lend;
  const uint32_t G = gridDim.x;
  const uint32_t first_li = begin + blockIdx.x;
  const uint32_t n_mine = first_li < lend ? (lend - first_li + G - 1) / G : 0;
  if (tid == 0) {
    for (int i = 0; i < TS; ++i) {
      mbar_init(&sm.full[i], 1);
      mbar_init(&sm.empty[i], 1);
    }
    for (int b = 0; b < TSLOT; ++b) {
      sm.slot_gen[b] = 0;
      sm.rq[b] = 0xFFFFFFF0u;  // (a lap tag no entry carries)
    }
    sm.rq_n = 0;
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (n_mine == 0) return;
  volatile uint32_t* vgen = sm.slot_gen;
  volatile uint32_t* vrq_n = &sm.rq_n;

  if (wid == 0) {  // ---------------------------------------------------------------- producer
    if (lane != 0) return;
    unsigned long long policy;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(policy));
    uint32_t seq = 0;  // stages issued
    auto issue = [&](uint32_t b, uint32_t pos, uint32_t n) {  // one stage: records [pos, pos + n)
      const uint32_t st = seq % TS, ph = (seq / TS) & 1u;
      mbar_wait(&sm.empty[st], ph ^ 1u);
      sm.st_slot[st] = b;
      sm.st_n[st] = n;
      sm.st_pos[st] = pos;
      const uint32_t n4 = (n + 3u) & ~3u;  // (extents and lists are 4-record aligned and padded)
      mbar_expect_tx(&sm.full[st], n4 * 12u);
      bulk_load(sm.obj[st], s.ar.obj + pos, n4 * 4u, &sm.full[st], policy);
      bulk_load(sm.key[st], s.ar.key + pos, n4 * 8u, &sm.full[st], policy);
      ++seq;
    };
    // Software pipeline over the CTA's cells: while cell j's pieces are issued, cell j+1's chain
    // head, cleaned list and first extent are already being loaded (each a dependent global round
    // trip: without this the ring drains at every cell boundary)
    struct Ext {
      uint32_t a, l, nxt, tm;
    };
    auto load_ext = [&](uint32_t e) {
      Ext x{0, 0, NONE, 0};
      if (is_extent(e)) x = Ext{s.x_start[e], s.x_len[e], s.x_next[e], s.x_tmax[e]};
      return x;
    };
    uint32_t c_cur = s.flush_list[first_li];
    uint32_t h_cur = s.cell_head[c_cur];
    uint2 comp_cur = s.cell_comp[c_cur];
    Ext x_cur = load_ext(h_cur);
    uint32_t c_nxt = n_mine > 1 ? s.flush_list[first_li + G] : 0;
    for (uint32_t j = 0; j < n_mine; ++j) {
      const uint32_t b = j % TSLOT;
      const uint32_t c = c_cur, head = h_cur;
      const uint2 comp = comp_cur;
      const Ext x0 = x_cur;
      // next cell's head and list, and the cell after's id
      uint32_t h_nxt = NONE;
      uint2 comp_nxt = make_uint2(0, 0);
      uint32_t c_nn = 0;
      if (j + 1 < n_mine) {
        h_nxt = s.cell_head[c_nxt];
        comp_nxt = s.cell_comp[c_nxt];
        if (j + 2 < n_mine) c_nn = s.flush_list[first_li + (j + 2) * G];
      }
      while (vgen[b] != j / TSLOT) __nanosleep(32);  // the slot's previous cell is indexed
      TSlot<WCAP>& sl = sm.slot[b];
      sl.c = c;
      sl.head = head;
      sl.comp = comp;
      sl.has = 1;
      sl.n_win = 0;
      sl.nrec = 0;
      sl.nexp = 0;
      sl.spill = spill + ((size_t)blockIdx.x * TSLOT + b) * spill_cap;
      sl.spill_cap = spill_cap;
      sl.state = 0;
      __threadfence_block();
      // walk the chain in segments of up to 16 extents: the pieces of every segment but the
      // last are issued before the total is known; the total is added before the last segment's
      uint32_t xs[16], xl[16];
      uint32_t e = head;
      bool first = true;
      unsigned long long issued = 0;
      unsigned long long nrec = 0, nexp = 0;
      bool done = false, prefetched = j + 1 >= n_mine;
      Ext x_nxt{0, 0, NONE, 0};
      while (!done) {
        uint32_t nx = 0;
        while (is_extent(e) && nx < 16) {
          const Ext x = first ? x0 : load_ext(e);
          first = false;
          if (t_cut && x.tm < t_cut) {
            nexp += x.l;
          } else if (x.l) {
            xs[nx] = x.a;
            xl[nx] = x.l;
            ++nx;
            nrec += x.l;
          }
          e = x.nxt;
        }
        const bool last_seg = !is_extent(e);
        if (last_seg && comp.y && nx < 16) {
          xs[nx] = comp.x;
          xl[nx] = comp.y;
          ++nx;
          nrec += comp.y;
          done = true;
        } else if (last_seg && !comp.y) {
          done = true;
        }
        unsigned long long pieces = 0;
        for (uint32_t x = 0; x < nx; ++x) pieces += (xl[x] + TCHUNK - 1) / TCHUNK;
        if (done) {  // the total first: the cell completes when the match warps catch up with it
          sl.nrec = nrec;
          sl.nexp = nexp;
          __threadfence_block();
          const unsigned long long total = issued + pieces;
          const unsigned long long old = atomicAdd(&sl.state, total << 32);
          if ((old & 0xFFFFFFFFull) == total) rq_push(&sm.rq_n, sm.rq, b);  // (all matched, or none)
        }
        for (uint32_t x = 0; x < nx; ++x)
          for (uint32_t o = 0; o < xl[x]; o += TCHUNK) {
            issue(b, xs[x] + o, min((uint32_t)TCHUNK, xl[x] - o));
            if (!prefetched) {  // (after the first piece: the next head has had a round trip)
              x_nxt = load_ext(h_nxt);
              prefetched = true;
            }
          }
        issued += pieces;
      }
      if (!prefetched) x_nxt = load_ext(h_nxt);  // (a cell with no pieces)
      c_cur = c_nxt;
      h_cur = h_nxt;
      comp_cur = comp_nxt;
      x_cur = x_nxt;
      c_nxt = c_nn;
    }
    for (int w = 0; w < TMW; ++w) {  // one sentinel stage per match warp: no more pieces
      const uint32_t st = seq % TS, ph = (seq / TS) & 1u;
      mbar_wait(&sm.empty[st], ph ^ 1u);
      sm.st_n[st] = 0xFFFFFFFFu;
      mbar_expect_tx(&sm.full[st], 0);
      ++seq;
    }
    return;
  }

  if (wid <= TMW) {  // ---------------------------------------------------------- match warps
    const unsigned long long* __restrict__ otk = s.ot_key;
    for (uint32_t seq = wid - 1;; seq += TMW) {
      const uint32_t st = seq % TS, ph = (seq / TS) & 1u;
      mbar_wait(&sm.full[st], ph);
      const uint32_t n = sm.st_n[st];
      if (n == 0xFFFFFFFFu) break;
      const uint32_t b = sm.st_slot[st], pos = sm.st_pos[st];
      TSlot<WCAP>& sl = sm.slot[b];
      // the stage in sub-pieces of 256 records (8 per lane in registers); the stage is released
      // once its last sub-piece is in registers
      constexpr int R = 8;
      constexpr int NSUB = TCHUNK / (32 * R);
      static_assert(TCHUNK % (32 * R) == 0, "pieces are whole sub-pieces of 256 records");
#pragma unroll 1
      for (int sub = 0; sub < NSUB; ++sub) {
        const uint32_t sb0 = (uint32_t)sub * 32 * R;
        uint32_t o[R];
        unsigned long long k[R], tg[R];
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const uint32_t i = sb0 + lane + 32 * r;
          o[r] = sm.obj[st][i];
          k[r] = sm.key[st][i];
        }
#pragma unroll
        for (int r = 0; r < R; ++r) tg[r] = (sb0 + lane + 32 * r) < n ? __ldg(otk + o[r]) : ~k[r];
        if (sub == NSUB - 1) {
          __syncwarp();
          if (lane == 0) mbar_arrive(&sm.empty[st]);  // (the stage's words are in registers now)
        }
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const bool hit = tg[r] == k[r];
          const unsigned hm = __ballot_sync(0xffffffffu, hit);
          if (hm) {
            uint32_t base = 0;
            if (lane == __ffs(hm) - 1) base = atomicAdd(&sl.n_win, (unsigned)__popc(hm));
            base = __shfl_sync(0xffffffffu, base, __ffs(hm) - 1);
            const uint32_t w = base + __popc(hm & lt);
            if (hit) {
              const uint32_t p = pos + sb0 + lane + 32 * r;
              if (w < (uint32_t)WCAP) sl.w_pos[w] = p;
              else if (w - (uint32_t)WCAP < sl.spill_cap) sl.spill[w - WCAP] = p;
            }
          }
        }
      }
      __syncwarp();
      if (lane == 0) {
        __threadfence_block();  // (the winners above before the piece counts as matched)
        const unsigned long long now = atomicAdd(&sl.state, 1ull) + 1ull;
        if ((now >> 32) != 0 && (now & 0xFFFFFFFFull) == (now >> 32)) rq_push(&sm.rq_n, sm.rq, b);
      }
    }
    return;
  }

  // ------------------------------------------------------------------------------- index warp
  (void)vrq_n;
  for (uint32_t j = 0; j < n_mine; ++j) {  // entry j of the queue (its lap tag says when it is in)
    uint32_t b = 0;
    if (lane == 0) {
      volatile uint32_t* vrq = sm.rq;
      uint32_t v;
      while (((v = vrq[j % TSLOT]) >> 4) != j / TSLOT) __nanosleep(32);
      b = v & 15u;
      __threadfence_block();
    }
    b = __shfl_sync(0xffffffffu, b, 0);
    TSlot<WCAP>& sl = sm.slot[b];
    index_cell<HCAP, WCAP>(sm, sl, g, s, out, out_top, full_vobj, lane, sl.spill, spill_cap, t_cut);
    __syncwarp();
    if (lane == 0) {
      __threadfence_block();
      vgen[b] = vgen[b] + 1;  // the producer may reuse the slot
    }
    __syncwarp();
  }
}

template <int HCAP, int WCAP>
int blocks_per_sm_t(bool tma);
template <int HCAP, int WCAP>
void launch_t(const DevGraph& g, const DevState& s, const Arena& out, unsigned long long* out_top,
              uint32_t begin, int full_vobj, int sm_count, uint32_t* spill, uint32_t spill_cap,
              uint32_t t_cut, uint32_t max_ctas, int mode, cudaStream_t st) {
  const bool tma = mode == FLUSH_TMA;
  cudaLaunchAttribute attr[1];
  if (mode == FLUSH_WARP) {  // warp-per-cell pass (the caller then runs k_flush over OVF_PASS)
    static int wbps[64] = {0};  // occupancy per device ordinal (set on first use)
    int dev = 0;
    cudaGetDevice(&dev);
    int& wb = wbps[dev & 63];
    if (!wb) {
      int b = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_flush_warp, FW * 32, 0);
      wb = std::max(b, 1);
    }
    uint32_t wgrid = (uint32_t)(sm_count * wb);
    if (max_ctas && max_ctas < wgrid) wgrid = max_ctas;
    const cudaLaunchConfig_t wcfg = pdl_config(dim3(wgrid), dim3(FW * 32), 0, st, attr);
    cudaLaunchKernelEx(&wcfg, k_flush_warp, g, s, out, out_top, begin, s.ovf_list, t_cut);
    return;
  }
  const int blocks_per_sm = blocks_per_sm_t<HCAP, WCAP>(tma);
  uint32_t grid = (uint32_t)(sm_count * blocks_per_sm);
  if (max_ctas && max_ctas < grid) grid = max_ctas;  // few cells to clean: fewer idle CTAs
  if (tma) {
    const cudaLaunchConfig_t cfg = pdl_config(dim3(grid), dim3(TFT), sizeof(TFlushSmem<HCAP, WCAP>), st, attr);
    cudaLaunchKernelEx(&cfg, k_flush_tma<HCAP, WCAP>, g, s, out, out_top, begin, full_vobj, spill, spill_cap, t_cut);
    return;
  }
  const cudaLaunchConfig_t cfg = pdl_config(dim3(grid), dim3(FT), sizeof(FlushSmem<HCAP, WCAP>), st, attr);
  cudaLaunchKernelEx(&cfg, k_flush<HCAP, WCAP>, g, s, out, out_top, begin, full_vobj, spill, spill_cap, t_cut);
}
template <int HCAP, int WCAP>
int blocks_per_sm_t(bool tma) {
  static int bps[2] = {0, 0};  // (occupancy: the same on every B200)
  int& blocks_per_sm = bps[tma ? 1 : 0];
  const int smem = tma ? (int)sizeof(TFlushSmem<HCAP, WCAP>) : (int)sizeof(FlushSmem<HCAP, WCAP>);
  if (tma) func_attr_once(k_flush_tma<HCAP, WCAP>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  else func_attr_once(k_flush<HCAP, WCAP>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (blocks_per_sm == 0) {
    int b = 0;
    if (tma) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_flush_tma<HCAP, WCAP>, TFT, smem);
    else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_flush<HCAP, WCAP>, FT, smem);
    blocks_per_sm = std::max(b, 1);
  }
  // ask for no more shared memory than the resident CTAs need: the rest stays L1, which
  // holds the object-table lines the match phase gathers (per device, like the size above)
  const int carve = std::min(100, (blocks_per_sm * (smem + 1024) * 100 + 228 * 1024 - 1) / (228 * 1024));
  if (tma) func_attr_once(k_flush_tma<HCAP, WCAP>, cudaFuncAttributePreferredSharedMemoryCarveout, carve);
  else func_attr_once(k_flush<HCAP, WCAP>, cudaFuncAttributePreferredSharedMemoryCarveout, carve);
  return blocks_per_sm;
}
}  // namespace

// the variant for a given cell size and average objects per cell: staging sized for ~2x the
// live objects of an average cell (more winners spill their positions to global memory)
static int flush_variant(uint32_t cs, uint32_t objects_per_cell) {
  const int h = cs <= 1024 ? 0 : 1;
  const int w = objects_per_cell <= 64 ? 0 : objects_per_cell <= 256 ? 1 : 2;
  return w * 2 + h;
}
static const uint32_t kWcap[3] = {128, 512, 2048};

size_t flush_spill_bytes(uint32_t cs, uint32_t objects_per_cell, int sm_count, uint32_t* cap) {
  const int v = flush_variant(cs, objects_per_cell);
  const uint32_t wcap = kWcap[v / 2];
  // room for 4x the average cell beyond the staging (a cell with more is re-streamed)
  uint32_t want = 0;
  if (4ull * objects_per_cell > wcap) {
    want = 1024;
    while (want < 4ull * objects_per_cell - wcap && want < (1u << 20)) want <<= 1;
  }
  *cap = want;
  if (!want) return 0;
  // (either kernel may run: room for the larger of their per-CTA spill areas)
  size_t per_sm = 0;
  for (int t = 0; t < 2; ++t) {
    int bps = 0;
    switch (v) {
      case 0: bps = blocks_per_sm_t<1024, 128>(t); break;
      case 1: bps = blocks_per_sm_t<4096, 128>(t); break;
      case 2: bps = blocks_per_sm_t<1024, 512>(t); break;
      case 3: bps = blocks_per_sm_t<4096, 512>(t); break;
      case 4: bps = blocks_per_sm_t<1024, 2048>(t); break;
      default: bps = blocks_per_sm_t<4096, 2048>(t); break;
    }
    per_sm = std::max(per_sm, (size_t)bps * (t ? TSLOT : NBUF));
  }
  return (size_t)sm_count * per_sm * want * sizeof(uint32_t);
}

void launch_flush(const DevGraph& g, const DevState& s, const Arena& out,
                  unsigned long long* out_top, uint32_t begin, uint32_t objects_per_cell,
                  int full_vobj, int sm_count, uint32_t* spill, uint32_t spill_cap, uint32_t t_cut,
                  uint32_t max_ctas, int mode, cudaStream_t st) {
  const int t = mode;
  switch (flush_variant(g.cs, objects_per_cell)) {
    case 0: launch_t<1024, 128>(g, s, out, out_top, begin, full_vobj, sm_count, spill, spill_cap, t_cut, max_ctas, t, st); break;
    case 1: launch_t<4096, 128>(g, s, out, out_top, begin, full_vobj, sm_count, spill, spill_cap, t_cut, max_ctas, t, st); break;
    case 2: launch_t<1024, 512>(g, s, out, out_top, begin, full_vobj, sm_count, spill, spill_cap, t_cut, max_ctas, t, st); break;
    case 3: launch_t<4096, 512>(g, s, out, out_top, begin, full_vobj, sm_count, spill, spill_cap, t_cut, max_ctas, t, st); break;
    case 4: launch_t<1024, 2048>(g, s, out, out_top, begin, full_vobj, sm_count, spill, spill_cap, t_cut, max_ctas, t, st); break;
    default: launch_t<4096, 2048>(g, s, out, out_top, begin, full_vobj, sm_count, spill, spill_cap, t_cut, max_ctas, t, st); break;
  }
}

}  // namespace gg

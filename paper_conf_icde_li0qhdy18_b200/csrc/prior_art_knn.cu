// prior_art_knn.cu — the paper's kNN query pipeline (Alg. 4-6, P@44429-52751) built on B200 as a
// comparison path (not used by ggrid_knn).
//
//   Alg. 4 l.1-4  candidate cells: L = c_q and its neighbour cells (P@47172); rings of
//                 neighbours are added until the cells hold >= rho k objects (reading R15: L
//                 grows by rings; it stops when no cell is new, or at PA_LMAX cells)
//   Alg. 5        GPU_SDist: Bellman-Ford over the vertices of L, relaxing every arc inside L
//                 until nothing changes (the paper repeats |V| times; the fixpoint is the same)
//   GPU_First_k   R_can = the k objects of L nearest by D[src(e_o)] + d_o (P@49436) and the
//                 same-arc term of reading R2; l = the k-th distance (unbounded if fewer)
//   Def. 3        GPU_Unresolved: vertices of L with an arc leaving L and D[v] <= l (inclusive,
//                 reading R13)
//   Alg. 6        Refine_kNN on CPU threads: from each unresolved v a Dijkstra bounded by
//                 l - D[v] over the whole graph, the objects met, per-object minimum (reading
//                 R14), first k of the union with R_can
// The message cleaning of L is an eager flush of every dirty cell before the batch (timed
// apart).  Per query the GPU phase is one CTA; queries go in waves of PA_WAVE CTAs (the
// per-query D array of |L| x cell_size words lives in global scratch).
#include <algorithm>
#include <atomic>
#include <chrono>
#include <queue>
#include <thread>
#include <unordered_map>

#include "handle.cuh"

namespace {

constexpr int PA_LMAX = 64;        // candidate cells per query
constexpr int PA_HASH = 256;       // cell -> slot table (shared memory)
constexpr uint32_t PA_CCAP = 4096; // candidate objects per query (block sort in shared memory)
constexpr uint32_t PA_UCAP = 8192; // unresolved vertices kept per query
constexpr uint32_t PA_WAVE = 2048; // queries per launch
constexpr int PA_T = 256;

struct PaQueryOut {
  uint32_t n_cells, n_vertices, iters, n_unres, l, flags;  // flags: 1 = candidate / unresolved cap hit
};

__device__ __forceinline__ int pa_slot(const uint32_t* hkey, const uint8_t* hval, uint32_t c) {
  uint32_t h = (c * 2654435761u) >> 24;  // 8 bits
  for (int p = 0; p < PA_HASH; ++p) {
    const uint32_t k = hkey[h];
    if (k == c) return hval[h];
    if (k == NONE) return -1;
    h = (h + 1) & (PA_HASH - 1);
  }
  return -1;
}

__global__ void __launch_bounds__(PA_T) k_pa_query(DevGraph g, DevState s, const uint2* __restrict__ q, uint32_t base,
                                                  uint32_t nq, uint32_t k, uint32_t rho_x100,
                                                  uint32_t* __restrict__ dscratch, uint32_t dstride,
                                                  unsigned long long* __restrict__ cand_out,
                                                  uint2* __restrict__ unres, PaQueryOut* __restrict__ qout) {
  __shared__ uint32_t L[PA_LMAX];
  __shared__ uint32_t nL, changed, ncand, nun;
  __shared__ uint32_t hkey[PA_HASH];
  __shared__ uint8_t hval[PA_HASH];
  __shared__ unsigned long long cand[PA_CCAP];
  const uint32_t qi = base + blockIdx.x;
  if (qi >= nq) return;
  const int tid = threadIdx.x;
  const uint2 qq = q[qi];
  const uint2 ei = g.einfo[qq.x];
  uint32_t* D = dscratch + (size_t)blockIdx.x * dstride;
  for (int i = tid; i < PA_HASH; i += PA_T) hkey[i] = NONE;
  __syncthreads();
  auto add_cell = [&](uint32_t c) {  // (thread 0)
    uint32_t h = (c * 2654435761u) >> 24;
    while (hkey[h] != NONE) {
      if (hkey[h] == c) return false;
      h = (h + 1) & (PA_HASH - 1);
    }
    if (nL >= PA_LMAX) return false;
    hkey[h] = c;
    hval[h] = (uint8_t)nL;
    L[nL++] = c;
    return true;
  };
  if (tid == 0) {  // ---- Alg. 4 lines 1-4
    nL = 0;
    const uint32_t cq = cellof(g, ei.x);
    add_cell(cq);
    for (uint32_t j = g.cadj_ptr[cq]; j < g.cadj_ptr[cq + 1]; ++j) add_cell(g.cadj[j]);
    uint64_t cnt = 0;
    for (uint32_t i = 0; i < nL; ++i) cnt += s.cell_comp[L[i]].y;
    uint32_t ring_lo = 0;
    while (cnt * 100 < (uint64_t)rho_x100 * k && nL < PA_LMAX) {
      const uint32_t ring_hi = nL;
      bool grew = false;
      for (uint32_t i = ring_lo; i < ring_hi && nL < PA_LMAX; ++i)
        for (uint32_t j = g.cadj_ptr[L[i]]; j < g.cadj_ptr[L[i] + 1]; ++j)
          if (add_cell(g.cadj[j])) {
            cnt += s.cell_comp[g.cadj[j]].y;
            grew = true;
          }
      ring_lo = ring_hi;
      if (!grew) break;
    }
    changed = 1;
    ncand = 0;
    nun = 0;
  }
  __syncthreads();
  const uint32_t nl = nL, cs = g.cs;
  const uint32_t nv = nl * cs;
  for (uint32_t i = tid; i < nv; i += PA_T) D[i] = INF;
  __syncthreads();
  auto dslot = [&](uint32_t v) -> int {  // index of vertex v in D, or -1 outside L
    const int sl = pa_slot(hkey, hval, cellof(g, v));
    return sl < 0 ? -1 : sl * (int)cs + (int)(v - cellof(g, v) * cs);
  };
  if (tid == 0) {  // seed (reading R1)
    if (qq.y == 0) D[dslot(ei.x)] = 0;
    else {
      const int d = dslot(g.edst[qq.x]);
      if (d >= 0) D[d] = ei.y - qq.y;
    }
  }
  __syncthreads();
  // ---- Alg. 5: relax every arc inside L until nothing changes
  uint32_t iters = 0;
  while (changed) {
    __syncthreads();
    if (tid == 0) changed = 0;
    __syncthreads();
    ++iters;
    for (uint32_t i = tid; i < nv; i += PA_T) {
      const uint32_t du = D[i];
      if (du == INF) continue;
      const uint32_t v = L[i / cs] * cs + i % cs;
      if (v >= g.V) continue;
      for (uint32_t a = g.rowptr[v]; a < g.rowptr[v + 1]; ++a) {
        const uint2 arc = g.adj[a];
        const int d = dslot(arc.x);
        if (d < 0) continue;
        const unsigned long long nd = (unsigned long long)du + arc.y;
        if (nd < D[d]) {
          atomicMin(&D[d], (uint32_t)nd);
          changed = 1;
        }
      }
    }
    __syncthreads();
  }
  // ---- GPU_First_k over the objects of L
  for (uint32_t ci = 0; ci < nl; ++ci) {
    const uint2 comp = s.cell_comp[L[ci]];
    for (uint32_t j = tid; j < comp.y; j += PA_T) {
      const uint32_t p = comp.x + j;
      const uint32_t ob = s.ar.obj[p], vs = s.ar.vsrc[p], off = s.ar.off[p], ed = s.ar.edge[p];
      const int d = dslot(vs);
      unsigned long long dist = (d >= 0 && D[d] != INF) ? (unsigned long long)D[d] + off : ~0ull;
      if (ed == qq.x && off >= qq.y) dist = min(dist, (unsigned long long)(off - qq.y));
      if (dist < INF) {
        const uint32_t i = atomicAdd(&ncand, 1u);
        if (i < PA_CCAP) cand[i] = (dist << 32) | ob;
      }
    }
  }
  __syncthreads();
  const uint32_t nc = min(ncand, PA_CCAP);
  // block bitonic sort of the candidates
  uint32_t n2 = 1;
  while (n2 < nc) n2 <<= 1;
  for (uint32_t i = nc + tid; i < n2; i += PA_T) cand[i] = ~0ull;
  __syncthreads();
  for (uint32_t size = 2; size <= n2; size <<= 1)
    for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
      for (uint32_t i = tid; i < n2 / 2; i += PA_T) {
        const uint32_t lo = 2 * i - (i & (stride - 1)), hi = lo + stride;
        const bool asc = (lo & size) == 0;
        const unsigned long long x = cand[lo], y = cand[hi];
        if ((x > y) == asc) {
          cand[lo] = y;
          cand[hi] = x;
        }
      }
      __syncthreads();
    }
  const uint32_t l = nc >= k ? (uint32_t)(cand[k - 1] >> 32) : INF;
  for (uint32_t r = tid; r < k; r += PA_T) cand_out[(size_t)qi * k + r] = r < nc ? cand[r] : ~0ull;
  // ---- Def. 3: unresolved vertices (an arc leaving L, D[v] <= l)
  for (uint32_t i = tid; i < nv; i += PA_T) {
    const uint32_t dv = D[i];
    if (dv == INF || dv > l) continue;
    const uint32_t v = L[i / cs] * cs + i % cs;
    if (v >= g.V) continue;
    bool edge = false;
    for (uint32_t a = g.rowptr[v]; a < g.rowptr[v + 1] && !edge; ++a) edge = dslot(g.adj[a].x) < 0;
    if (edge) {
      const uint32_t j = atomicAdd(&nun, 1u);
      if (j < PA_UCAP) unres[(size_t)qi * PA_UCAP + j] = make_uint2(v, dv);
    }
  }
  __syncthreads();
  if (tid == 0)
    qout[qi] = PaQueryOut{nl, nv, iters, min(nun, PA_UCAP), l, (ncand > PA_CCAP || nun > PA_UCAP) ? 1u : 0u};
}

// every cell's cleaned list, compacted: (obj, vsrc, off) per object, in cell order
__global__ void k_pa_lists(DevGraph g, DevState s, const uint32_t* __restrict__ off, uint4* __restrict__ out) {
  const uint32_t c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= g.n_cells) return;
  const uint2 comp = s.cell_comp[c];
  uint32_t o = off[c];
  for (uint32_t j = 0; j < comp.y; ++j) {
    const uint32_t p = comp.x + j;
    out[o++] = make_uint4(s.ar.obj[p], s.ar.vsrc[p], s.ar.off[p], 0);
  }
}
// the unresolved vertices of every query, compacted (offsets from the host)
__global__ void k_pa_compact_unres(const uint2* __restrict__ unres, const PaQueryOut* __restrict__ qo,
                                   const unsigned long long* __restrict__ off, uint32_t nq, uint2* __restrict__ out) {
  const uint32_t i = blockIdx.x;
  if (i >= nq) return;
  const uint32_t n = qo[i].n_unres;
  for (uint32_t j = threadIdx.x; j < n; j += blockDim.x) out[off[i] + j] = unres[(size_t)i * PA_UCAP + j];
}
__global__ void k_pa_list_counts(DevGraph g, DevState s, uint32_t* __restrict__ cnt) {
  const uint32_t c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c <= g.n_cells) cnt[c] = c < g.n_cells ? s.cell_comp[c].y : 0;
}

}  // namespace

extern "C" int ggrid_prior_art_knn(ggrid_t h, const ggrid_query* q, uint32_t n_q, uint32_t k, uint32_t rho_x100,
                                   uint32_t threads, uint32_t* out_obj, uint32_t* out_dist,
                                   ggrid_prior_art_knn_result* res) {
  if (!h || h->multi || k == 0 || k > PA_CCAP || rho_x100 < 100 || !q || !out_obj || !out_dist) return GGRID_EINVAL;
  using clk = std::chrono::steady_clock;
  auto ms = [](clk::time_point a, clk::time_point b) { return std::chrono::duration<double, std::milli>(b - a).count(); };
  CK(cudaSetDevice(h->device));
  cudaStream_t st = h->stream;
  ggrid_prior_art_knn_result r{};
  // ---- message cleaning of every dirty cell (Alg. 4 l.2, eagerly), timed apart
  RC(h->sync());
  auto t0 = clk::now();
  RC(ggrid_flush_all(h));
  auto t1 = clk::now();
  r.ms_clean = ms(t0, t1);
  const DevGraph& g = h->g;
  const DevState& s = h->s;
  // ---- host copies for Refine_kNN: the out-arc CSR and a vertex -> objects index
  if (h->pa_rowptr.empty()) {
    h->pa_rowptr.resize((size_t)h->V + 1);
    CK(cudaMemcpy(h->pa_rowptr.data(), g.rowptr, ((size_t)h->V + 1) * 4, cudaMemcpyDeviceToHost));
    h->pa_adj.resize(h->pa_rowptr.back());
    if (!h->pa_adj.empty())
      CK(cudaMemcpy(h->pa_adj.data(), g.adj, h->pa_adj.size() * 8, cudaMemcpyDeviceToHost));
  }
  DBuf cnt, off, scan_tmp, lists, dq, dsc, dcand, dunres, dqout;
  auto release = [&] {
    for (DBuf* b : {&cnt, &off, &scan_tmp, &lists, &dq, &dsc, &dcand, &dunres, &dqout}) b->release();
  };
  auto fail = [&](int rc) {
    release();
    return rc;
  };
  const uint32_t nc1 = h->n_cells + 1;
  const size_t sb = prior_art_scan_bytes(nc1);
  if (cnt.ensure(nc1 * 4) || off.ensure(nc1 * 4) || scan_tmp.ensure(sb)) return fail(GGRID_ENOMEM);
  k_pa_list_counts<<<(nc1 + 255) / 256, 256, 0, st>>>(g, s, cnt.as<uint32_t>());
  if (launch_pa_scan(scan_tmp.p, sb, cnt.as<uint32_t>(), off.as<uint32_t>(), nc1, st)) return fail(GGRID_ECUDA);
  uint32_t n_objs = 0;
  CK(cudaMemcpyAsync(&n_objs, off.as<uint32_t>() + h->n_cells, 4, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (lists.ensure((size_t)std::max(1u, n_objs) * 16)) return fail(GGRID_ENOMEM);
  k_pa_lists<<<(h->n_cells + 255) / 256, 256, 0, st>>>(g, s, off.as<uint32_t>(), lists.as<uint4>());
  std::vector<uint4> objs(n_objs);
  if (n_objs) CK(cudaMemcpyAsync(objs.data(), lists.p, (size_t)n_objs * 16, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  std::vector<uint32_t> vptr((size_t)h->V + 1, 0);
  std::vector<uint2> vobj(n_objs);  // (obj, off) grouped by source vertex
  for (const uint4& o : objs) vptr[o.y + 1]++;
  for (uint32_t v = 0; v < h->V; ++v) vptr[v + 1] += vptr[v];
  {
    std::vector<uint32_t> fill(vptr.begin(), vptr.end() - 1);
    for (const uint4& o : objs) vobj[fill[o.y]++] = make_uint2(o.x, o.z);
  }
  auto t2 = clk::now();
  r.ms_host_index = ms(t1, t2);
  // ---- GPU phase (Alg. 4 l.5-9) in waves of PA_WAVE queries
  const uint32_t dstride = PA_LMAX * h->cs;
  const uint32_t wave = std::min<uint32_t>(PA_WAVE, n_q);
  if (dq.ensure((size_t)n_q * 8) || dsc.ensure((size_t)wave * dstride * 4) || dcand.ensure((size_t)n_q * k * 8) ||
      dunres.ensure((size_t)n_q * PA_UCAP * 8) || dqout.ensure((size_t)n_q * sizeof(PaQueryOut)))
    return fail(GGRID_ENOMEM);
  CK(cudaMemcpyAsync(dq.p, q, (size_t)n_q * 8, cudaMemcpyDefault, st));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  CK(cudaEventRecord(e0, st));
  for (uint32_t b = 0; b < n_q; b += wave)
    k_pa_query<<<std::min(wave, n_q - b), PA_T, 0, st>>>(g, s, dq.as<uint2>(), b, n_q, k, rho_x100, dsc.as<uint32_t>(),
                                                         dstride, dcand.as<unsigned long long>(), dunres.as<uint2>(),
                                                         dqout.as<PaQueryOut>());
  CK(cudaEventRecord(e1, st));
  std::vector<unsigned long long> hcand((size_t)n_q * k);
  std::vector<PaQueryOut> hq(n_q);
  CK(cudaStreamSynchronize(st));
  float gms = 0.f;
  cudaEventElapsedTime(&gms, e0, e1);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  CK(cudaGetLastError());
  r.ms_gpu = gms;
  auto t3 = clk::now();
  CK(cudaMemcpy(hcand.data(), dcand.p, hcand.size() * 8, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(hq.data(), dqout.p, hq.size() * sizeof(PaQueryOut), cudaMemcpyDeviceToHost));
  uint64_t n_unres = 0;
  for (const PaQueryOut& x : hq) {
    n_unres += x.n_unres;
    r.cells += x.n_cells;
    r.vertices += x.n_vertices;
    r.bf_iterations += x.iters;
    if (x.flags) return fail(GGRID_ENOMEM);  // (a candidate or unresolved cap: not this tool's range)
  }
  // the unresolved lists, compacted on the device and copied once
  std::vector<unsigned long long> uoff(n_q + 1, 0);
  for (uint32_t i = 0; i < n_q; ++i) uoff[i + 1] = uoff[i] + hq[i].n_unres;
  std::vector<uint2> hun(std::max<unsigned long long>(1, uoff[n_q]));
  {
    DBuf doff, dcomp;
    if (doff.ensure((size_t)(n_q + 1) * 8) || dcomp.ensure(hun.size() * 8)) return fail(GGRID_ENOMEM);
    CK(cudaMemcpyAsync(doff.p, uoff.data(), (size_t)(n_q + 1) * 8, cudaMemcpyHostToDevice, st));
    k_pa_compact_unres<<<n_q, 128, 0, st>>>(dunres.as<uint2>(), dqout.as<PaQueryOut>(),
                                            doff.as<unsigned long long>(), n_q, dcomp.as<uint2>());
    if (uoff[n_q]) CK(cudaMemcpyAsync(hun.data(), dcomp.p, uoff[n_q] * 8, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    doff.release();
    dcomp.release();
  }
  auto t4 = clk::now();
  r.ms_d2h = ms(t3, t4);
  r.unresolved = n_unres;
  // ---- Alg. 6 Refine_kNN on CPU threads (one query per task; Dijkstra per unresolved vertex)
  const unsigned nt = threads ? threads : std::max(1u, std::thread::hardware_concurrency());
  std::atomic<uint32_t> next{0};
  std::atomic<uint64_t> settled{0};
  auto worker = [&] {
    std::unordered_map<uint32_t, uint64_t> dist;  // (a bounded search touches a small ball)
    std::vector<std::pair<uint64_t, uint32_t>> best;
    uint64_t n_settled = 0;
    for (;;) {
      const uint32_t i = next.fetch_add(1);
      if (i >= n_q) break;
      const uint64_t l = hq[i].l;  // INF (2^32-1) when fewer than k candidates: unbounded
      best.clear();
      for (uint32_t j = 0; j < k; ++j) {
        const unsigned long long c = hcand[(size_t)i * k + j];
        if (c != ~0ull) best.push_back({c >> 32, (uint32_t)c});
      }
      for (uint32_t u = 0; u < hq[i].n_unres; ++u) {
        const uint2 uv = hun[uoff[i] + u];
        const uint64_t radius = l - uv.y;  // dist(v, .) <= l - dist(q, v)
        using Item = std::pair<uint64_t, uint32_t>;
        std::priority_queue<Item, std::vector<Item>, std::greater<Item>> pq;
        dist.clear();
        dist[uv.x] = 0;
        pq.push({0, uv.x});
        while (!pq.empty()) {
          const Item it = pq.top();
          pq.pop();
          if (it.first != dist[it.second]) continue;
          ++n_settled;
          const uint32_t x = it.second;
          for (uint32_t j = vptr[x]; j < vptr[x + 1]; ++j) {
            const uint64_t d = (uint64_t)uv.y + it.first + vobj[j].y;
            if (d <= l && d < 0xFFFFFFFFull) best.push_back({d, vobj[j].x});
          }
          for (uint32_t a = h->pa_rowptr[x]; a < h->pa_rowptr[x + 1]; ++a) {
            const uint2 arc = h->pa_adj[a];
            const uint64_t nd = it.first + arc.y;
            if (nd > radius) continue;
            auto f = dist.find(arc.x);
            if (f == dist.end() || nd < f->second) {
              dist[arc.x] = nd;
              pq.push({nd, arc.x});
            }
          }
        }
      }
      // per-object minimum (reading R14), then the first k by (dist, obj)
      std::sort(best.begin(), best.end(), [](const std::pair<uint64_t, uint32_t>& a, const std::pair<uint64_t, uint32_t>& b) {
        return a.second != b.second ? a.second < b.second : a.first < b.first;
      });
      best.erase(std::unique(best.begin(), best.end(),
                             [](const std::pair<uint64_t, uint32_t>& a, const std::pair<uint64_t, uint32_t>& b) {
                               return a.second == b.second;
                             }),
                 best.end());
      std::sort(best.begin(), best.end());
      for (uint32_t j = 0; j < k; ++j) {
        const bool ok = j < best.size();
        out_obj[(size_t)i * k + j] = ok ? best[j].second : GGRID_PAD;
        out_dist[(size_t)i * k + j] = ok ? (uint32_t)best[j].first : GGRID_PAD;
      }
    }
    settled += n_settled;
  };
  std::vector<std::thread> pool;
  for (unsigned t = 1; t < nt; ++t) pool.emplace_back(worker);
  worker();
  for (auto& t : pool) t.join();
  auto t5 = clk::now();
  r.ms_cpu_refine = ms(t4, t5);
  r.refine_settled = settled;
  r.threads = nt;
  if (res) *res = r;
  release();
  return GGRID_OK;
}

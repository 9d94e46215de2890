// api.cu — the C ABI (include/ggrid.h): host-side graph-grid build, device memory
// management, ingest / knn orchestration, garbage collection of the record arena.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <new>
#include <tuple>
#include <utility>
#include <vector>

#include "handle.cuh"


namespace gg {
cudaError_t func_attr_once(const void* kernel, cudaFuncAttribute attr, int value) {
  static std::mutex mu;
  static std::map<std::tuple<const void*, int, int, int>, cudaError_t> done;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return cudaGetLastError();
  std::lock_guard<std::mutex> lock(mu);
  const auto key = std::make_tuple(kernel, (int)attr, dev, value);
  auto it = done.find(key);
  if (it != done.end()) return it->second;
  const cudaError_t e = cudaFuncSetAttribute(kernel, attr, value);
  if (e != cudaSuccess) cudaGetLastError();
  done[key] = e;
  return e;
}
}  // namespace gg

// ------------------------------------------------------------------------------------------
// Garbage collection of the log arena: every cell (clean or not) is cleaned into a fresh
// arena, which is copied back to the start of the main one; the extent pool is emptied.
int ggrid_s::gc() {
  RC(sync());
  const uint64_t live = (uint64_t)h_status->n_live + 4ull * n_cells + 16;
  const size_t per = 4 + 8 + 4 + 4 + 4;
  RC(gc_buf.ensure(live * per + 64));
  Arena t;
  unsigned char* b = gc_buf.as<unsigned char>();
  t.key = reinterpret_cast<unsigned long long*>(b);
  t.obj = reinterpret_cast<uint32_t*>(t.key + live);
  t.vsrc = t.obj + live;
  t.off = t.vsrc + live;
  t.edge = t.off + live;
  t.cap = live;
  unsigned long long* d_top = nullptr;
  RC(misc.ensure(64));
  d_top = misc.as<unsigned long long>();
  epoch++;
  {
    WordSet ws;
    ws.zero_range(reinterpret_cast<uint32_t*>(d_top), 2);
    ws.add(&d_status->n_flush, 0);
    RC(set_words(ws));
  }
  launch(GGRID_K_OTHER, [&] { launch_mark_dirty(g, s, epoch, 1, stream); });
  RC(flush_list_run(t, d_top, 0, /*full_vobj=*/1));
  unsigned long long top = 0;
  CK(cudaMemcpyAsync(&top, d_top, 8, cudaMemcpyDeviceToHost, stream));
  RC(sync());
  if (h_status->err & ERR_ARENA) return GGRID_ENOMEM;
  CK(cudaMemcpyAsync(s.ar.obj, t.obj, top * 4, cudaMemcpyDeviceToDevice, stream));
  CK(cudaMemcpyAsync(s.ar.key, t.key, top * 8, cudaMemcpyDeviceToDevice, stream));
  CK(cudaMemcpyAsync(s.ar.vsrc, t.vsrc, top * 4, cudaMemcpyDeviceToDevice, stream));
  CK(cudaMemcpyAsync(s.ar.off, t.off, top * 4, cudaMemcpyDeviceToDevice, stream));
  CK(cudaMemcpyAsync(s.ar.edge, t.edge, top * 4, cudaMemcpyDeviceToDevice, stream));
  CK(cudaMemcpyAsync(&d_status->arena_top, &top, 8, cudaMemcpyHostToDevice, stream));
  RC(set_status_u32(&d_status->ext_top, 0));
  RC(sync());
  // gc_buf stays allocated (live-sized, small next to the arena): a cudaMalloc/cudaFree pair
  // per collection costs milliseconds and synchronises the device
  stats.gc_runs++;
  return GGRID_OK;
}

// Re-basing of the arrival index (a sustained update stream, §8(f) N1: P@53218 "we can safely
// delete the messages before t_now - t_Delta").  Only the ORDER of keys matters (the validity
// test is key == ot_key[obj], and ot_key is a max).  After a garbage collection every live
// object has at most one record left, the one whose key equals its ot_key (GC keeps exactly
// the winners).  Rewriting every key k != 0 as (k & ~0xFFFFFFFF) | 1 in the arena AND in ot_key
// therefore keeps every equality, and keeps every existing key below any later update's key
// (t, seq >= 2) with the same t -- later arrivals still win ties (reading R7).
int ggrid_s::rebase() {
  RC(gc());  // (syncs: no ingest batch is in flight)
  launch(GGRID_K_OTHER, [&] { launch_rebase_keys(s, h_status->arena_top, stream); });
  RC(sync());
  seq_next = 2;
  rebases++;
  return GGRID_OK;
}

int ggrid_s::ensure_arena(uint64_t need_records, uint32_t need_ext) {
  const bool fits_a = h_status->arena_top + pend_records + need_records <= s.ar.cap;
  const bool fits_e = (uint64_t)h_status->ext_top + pend_ext + need_ext <= s.ext_cap;
  if (fits_a && fits_e) return GGRID_OK;
  RC(gc());  // (syncs first: the pending bounds are resolved)
  if (h_status->arena_top + need_records > s.ar.cap) return GGRID_ENOMEM;
  if ((uint64_t)h_status->ext_top + need_ext > s.ext_cap) return GGRID_ENOMEM;
  return GGRID_OK;
}

// ------------------------------------------------------------------------------------------
static int build_one(const ggrid_graph* gr, uint32_t cell_size, const ggrid_opts& opts_in, ggrid_t* out);

// a call on the front handle of an in-process multi-GPU index, applied to every shard in turn
template <class F>
static int each_shard(ggrid_t h, F&& f) {
  for (uint32_t r = 0; r < multi_n(h->multi); ++r) RC(f(multi_shard(h->multi, (int)r)));
  return GGRID_OK;
}
#define SINGLE_ONLY(h) \
  do {                 \
    if ((h) && (h)->multi) return GGRID_EINVAL; \
  } while (0)

extern "C" {

const char* ggrid_version(void) { return "ggrid-b200 0.1 (sm_100a)"; }

const char* ggrid_strerror(int rc) {
  switch (rc) {
    case GGRID_OK: return "ok";
    case GGRID_EINVAL: return "invalid argument";
    case GGRID_ENOMEM: return "out of memory";
    case GGRID_ECUDA: return "CUDA error";
    case GGRID_ENCCL: return "NCCL error";
    case GGRID_EOVERFLOW: return "arrival index overflow (more than 2^32 updates)";
    default: return "unknown error";
  }
}

uint64_t ggrid_zvalue(uint32_t x, uint32_t y) {
  uint64_t z = 0;
  for (int b = 0; b < 32; ++b) {
    z |= (uint64_t)((x >> b) & 1u) << (2 * b);
    z |= (uint64_t)((y >> b) & 1u) << (2 * b + 1);
  }
  return z;
}

int ggrid_build(const ggrid_graph* gr, uint32_t cell_size, const ggrid_opts* opts, ggrid_t* out) {
  if (!gr || !out) return GGRID_EINVAL;
  *out = nullptr;
  ggrid_opts o{};
  if (opts) o = *opts;
  if (o.exchange_kind > GGRID_EXCHANGE_NCCL) return GGRID_EINVAL;
  if (o.n_gpus > 1) {
    if (o.n_ranks > 1) return GGRID_EINVAL;  // (one process drives all shards, or one each)
    return multi_build(gr, cell_size, o, out, build_one);
  }
  ggrid_t h = nullptr;
  RC(build_one(gr, cell_size, o, &h));
  if (o.n_ranks > 1) {
    const int rc = rank_attach(h, o);
    if (rc != GGRID_OK) {
      ggrid_free(h);
      return rc;
    }
  }
  *out = h;
  return GGRID_OK;
}

}  // extern "C"

static int build_one(const ggrid_graph* gr, uint32_t cell_size, const ggrid_opts& opts_in, ggrid_t* out) {
  const ggrid_opts* opts = &opts_in;
  *out = nullptr;
  const uint32_t V = gr->n_vertices, A = gr->n_arcs;
  if (V == 0 || V >= 0xFFFFFFFEu || A >= 0xFFFFFFFEu || cell_size == 0) return GGRID_EINVAL;
  if (A > 0 && (!gr->src || !gr->dst || !gr->w)) return GGRID_EINVAL;
  if ((gr->x == nullptr) != (gr->y == nullptr)) return GGRID_EINVAL;
  for (uint32_t a = 0; a < A; ++a)
    if (gr->src[a] >= V || gr->dst[a] >= V || gr->w[a] == 0) return GGRID_EINVAL;
  ggrid_opts o{};
  if (opts) o = *opts;
  if (o.max_k == 0) o.max_k = 256;
  if (o.max_k > expand_max_k(expand_levels() - 1)) return GGRID_EINVAL;
  if (o.max_objects == 0) o.max_objects = 1u << 24;
  if (o.max_objects == 0xFFFFFFFFu) return GGRID_EINVAL;
  if (o.log_capacity == 0) o.log_capacity = 1ull << 26;
  if (o.log_capacity > 0xFFFFFFF0ull) return GGRID_EINVAL;

  ggrid_s* h = new (std::nothrow) ggrid_s();
  if (!h) return GGRID_ENOMEM;
  auto fail = [&](int rc) {
    ggrid_free(h);
    return rc;
  };
  if (o.device > 0) {
    if (cudaSetDevice(o.device) != cudaSuccess) return fail(GGRID_ECUDA);
  }
  if (cudaGetDevice(&h->device) != cudaSuccess) return fail(GGRID_ECUDA);
  cudaDeviceGetAttribute(&h->sm_count, cudaDevAttrMultiProcessorCount, h->device);
  if (o.stream) {
    h->stream = (cudaStream_t)o.stream;
  } else {
    if (cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking) != cudaSuccess)
      return fail(GGRID_ECUDA);
    h->own_stream = true;
  }
  if (cudaStreamCreateWithFlags(&h->copy_stream, cudaStreamNonBlocking) != cudaSuccess) {
    return fail(GGRID_ECUDA);
  }
  if (cudaEventCreateWithFlags(&h->ev_in, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&h->ev_out, cudaEventDisableTiming) != cudaSuccess)
    return fail(GGRID_ECUDA);
  h->V = V;
  h->A = A;
  h->cs = cell_size;
  h->n_cells = (uint32_t)((V + (uint64_t)cell_size - 1) / cell_size);
  h->max_k = o.max_k;
  h->max_objects = o.max_objects;
  h->seed_neighbors = o.seed_neighbors == 2 ? 0 : 1;
  h->profile = o.profile;
  h->t_delta = o.t_delta;
  // the expiry cut reads t_now on the host, so expiry keeps ingest synchronous
  h->async_ingest = (o.async_ingest && !o.t_delta) ? 1 : 0;
  h->ingest_mode = o.ingest_kernels <= 4 ? (int)o.ingest_kernels : 0;
  if (const char* fk = getenv("GGRID_FLUSH_KERNEL")) h->flush_kernel = atoi(fk);  // (experiment hook)
  h->s.n_ranks = 1;
  h->s.rank = 0;

  // ---- graph grid: Z-order of quantised coordinates, cells = runs of cell_size vertices
  std::vector<uint32_t> order(V);
  for (uint32_t v = 0; v < V; ++v) order[v] = v;
  if (gr->x) {
    int64_t mnx = INT64_MAX, mxx = INT64_MIN, mny = INT64_MAX, mxy = INT64_MIN;
    for (uint32_t v = 0; v < V; ++v) {
      mnx = std::min<int64_t>(mnx, gr->x[v]);
      mxx = std::max<int64_t>(mxx, gr->x[v]);
      mny = std::min<int64_t>(mny, gr->y[v]);
      mxy = std::max<int64_t>(mxy, gr->y[v]);
    }
    const int64_t sx = std::max<int64_t>(1, mxx - mnx), sy = std::max<int64_t>(1, mxy - mny);
    std::vector<uint64_t> key(V);
    for (uint32_t v = 0; v < V; ++v) {
      uint32_t qx = (uint32_t)(((int64_t)gr->x[v] - mnx) * 65535 / sx);
      uint32_t qy = (uint32_t)(((int64_t)gr->y[v] - mny) * 65535 / sy);
      key[v] = (ggrid_zvalue(qx, qy) << 32) | v;
    }
    std::sort(key.begin(), key.end());
    for (uint32_t i = 0; i < V; ++i) order[i] = (uint32_t)key[i];
  }
  std::vector<uint32_t> newid(V);
  for (uint32_t i = 0; i < V; ++i) newid[order[i]] = i;
  h->user_cell.resize(V);
  for (uint32_t v = 0; v < V; ++v) h->user_cell[v] = newid[v] / cell_size;

  // ---- CSR over internal ids, inverted index (user edge -> src, w, dst).  An arc of weight
  // 2^32-1 can never lie on a path shorter than INF (R18), so it is left out of the CSR (its
  // inverted-index entry stays: objects and queries on it are still valid locations).
  constexpr uint32_t WMAX = 0xFFFFFFFFu;
  std::vector<uint32_t> rowptr((size_t)V + 1, 0);
  for (uint32_t a = 0; a < A; ++a)
    if (gr->w[a] != WMAX) rowptr[newid[gr->src[a]] + 1]++;
  for (uint32_t v = 0; v < V; ++v) rowptr[v + 1] += rowptr[v];
  const uint32_t An = rowptr[V];
  std::vector<uint2> adj(An), einfo(A);
  std::vector<uint32_t> edst(A);
  {
    std::vector<uint32_t> fill(rowptr.begin(), rowptr.end() - 1);
    uint64_t wsum = 0;
    for (uint32_t a = 0; a < A; ++a) {
      const uint32_t u = newid[gr->src[a]], v = newid[gr->dst[a]];
      if (gr->w[a] != WMAX) adj[fill[u]++] = make_uint2(v, gr->w[a]);
      einfo[a] = make_uint2(u, gr->w[a]);
      edst[a] = v;
      wsum += gr->w[a];
    }
    h->delta = o.delta ? o.delta : (uint32_t)std::max<uint64_t>(1, A ? wsum / A : 1);
  }
  // ---- inline adjacency: 4 slots (dst, w) per vertex, one 32-byte record, so the expansion
  // reads a vertex's arcs with one dependent load (road graphs: degree <= 4 almost always).
  // w = 0: empty slot; a vertex with more than 4 arcs keeps 3 inline and slot 3 = (u, WMAX):
  // "arcs 3.. of u are adj[rowptr[u]+3 .. rowptr[u+1])".
  std::vector<uint2> vadj((size_t)V * 4, make_uint2(0, 0));
  for (uint32_t u = 0; u < V; ++u) {
    const uint32_t d = rowptr[u + 1] - rowptr[u];
    const uint32_t inl = d <= 4 ? d : 3;
    for (uint32_t j = 0; j < inl; ++j) vadj[(size_t)u * 4 + j] = adj[rowptr[u] + j];
    if (d > 4) vadj[(size_t)u * 4 + 3] = make_uint2(u, WMAX);
  }
  // ---- cell adjacency (P@47172: c_i neighbours c_j if an arc goes from c_i to c_j)
  std::vector<uint64_t> cpairs;
  for (uint32_t a = 0; a < A; ++a) {
    const uint32_t cu = einfo[a].x / cell_size, cv = edst[a] / cell_size;
    if (cu != cv) cpairs.push_back(((uint64_t)cu << 32) | cv);
  }
  std::sort(cpairs.begin(), cpairs.end());
  cpairs.erase(std::unique(cpairs.begin(), cpairs.end()), cpairs.end());
  std::vector<uint32_t> cptr((size_t)h->n_cells + 1, 0), cadj(cpairs.size());
  for (size_t i = 0; i < cpairs.size(); ++i) {
    cptr[(cpairs[i] >> 32) + 1]++;
    cadj[i] = (uint32_t)cpairs[i];
  }
  for (uint32_t c = 0; c < h->n_cells; ++c) {
    h->max_cell_degree = std::max(h->max_cell_degree, cptr[c + 1]);
    cptr[c + 1] += cptr[c];
  }

  // ---- device graph
  uint32_t *d_rowptr, *d_edst, *d_cptr, *d_cadj;
  uint2 *d_adj, *d_einfo, *d_vadj;
  int rc;
  if ((rc = h->alloc(&d_rowptr, (size_t)V + 1, false))) return fail(rc);
  if ((rc = h->alloc(&d_adj, An, false))) return fail(rc);
  if ((rc = h->alloc(&d_vadj, (size_t)V * 4, false))) return fail(rc);
  if ((rc = h->alloc(&d_einfo, A, false))) return fail(rc);
  if ((rc = h->alloc(&d_edst, A, false))) return fail(rc);
  if ((rc = h->alloc(&d_cptr, (size_t)h->n_cells + 1, false))) return fail(rc);
  if ((rc = h->alloc(&d_cadj, cadj.size(), false))) return fail(rc);
  if (cudaMemcpy(d_rowptr, rowptr.data(), rowptr.size() * 4, cudaMemcpyHostToDevice) ||
      (An && cudaMemcpy(d_adj, adj.data(), (size_t)An * 8, cudaMemcpyHostToDevice)) ||
      cudaMemcpy(d_vadj, vadj.data(), vadj.size() * 8, cudaMemcpyHostToDevice) ||
      cudaMemcpy(d_einfo, einfo.data(), (size_t)A * 8, cudaMemcpyHostToDevice) ||
      cudaMemcpy(d_edst, edst.data(), (size_t)A * 4, cudaMemcpyHostToDevice) ||
      cudaMemcpy(d_cptr, cptr.data(), cptr.size() * 4, cudaMemcpyHostToDevice) ||
      (cadj.size() && cudaMemcpy(d_cadj, cadj.data(), cadj.size() * 4, cudaMemcpyHostToDevice)))
    return fail(GGRID_ECUDA);
  uint32_t cs_mul, cs_shift;
  fastdiv_params(cell_size, cs_mul, cs_shift);
  h->g = DevGraph{V,      A,       cell_size, h->n_cells, h->delta, cs_mul, cs_shift, d_rowptr,
                  d_adj,  d_einfo, d_edst,    d_cptr,     d_cadj,   d_vadj};

  // ---- dynamic state
  DevState& s = h->s;
  s.max_objects = o.max_objects;
  if ((rc = h->alloc(&s.ot_key, o.max_objects))) return fail(rc);
  const uint64_t cap = (o.log_capacity + 3) & ~3ull;
  s.ar.cap = cap;
  if ((rc = h->alloc(&s.ar.obj, cap + 4, false))) return fail(rc);
  if ((rc = h->alloc(&s.ar.key, cap + 4, false))) return fail(rc);
  if ((rc = h->alloc(&s.ar.vsrc, cap + 4, false))) return fail(rc);
  if ((rc = h->alloc(&s.ar.off, cap + 4, false))) return fail(rc);
  if ((rc = h->alloc(&s.ar.edge, cap + 4, false))) return fail(rc);
  s.ext_cap = (uint32_t)std::min<uint64_t>(std::max<uint64_t>(1u << 20, 16ull * h->n_cells), 1u << 27);
  if ((rc = h->alloc(&s.x_start, s.ext_cap, false))) return fail(rc);
  if ((rc = h->alloc(&s.x_len, s.ext_cap, false))) return fail(rc);
  if ((rc = h->alloc(&s.x_next, s.ext_cap, false))) return fail(rc);
  if ((rc = h->alloc(&s.x_tmax, s.ext_cap, false))) return fail(rc);
  if ((rc = h->alloc(&s.cell_head, h->n_cells, false))) return fail(rc);
  if (cudaMemset(s.cell_head, 0xFF, (size_t)h->n_cells * 4)) return fail(GGRID_ECUDA);
  if ((rc = h->alloc(&s.cell_pending, h->n_cells))) return fail(rc);
  if ((rc = h->alloc(&s.listed_cell, o.max_objects, false))) return fail(rc);
  if (cudaMemset(s.listed_cell, 0xFF, (size_t)o.max_objects * 4)) return fail(GGRID_ECUDA);
  if ((rc = h->alloc(&s.cell_req, h->n_cells))) return fail(rc);
  if ((rc = h->alloc(&s.v_obj, V))) return fail(rc);
  if ((rc = h->alloc(&s.vhas, (size_t)V / 32 + 2))) return fail(rc);
  if ((rc = h->alloc(&s.cell_comp, h->n_cells))) return fail(rc);
  s.vcnt = nullptr;
  if (cell_size > 4096 && (rc = h->alloc(&s.vcnt, V))) return fail(rc);
  if ((rc = h->alloc(&s.bcount, (size_t)h->n_cells * BCOUNT_STRIDE))) return fail(rc);
  if ((rc = h->alloc(&s.bbase, h->n_cells))) return fail(rc);
  if ((rc = h->alloc(&s.flush_list, h->n_cells))) return fail(rc);
  if ((rc = h->alloc(&s.ovf_list, h->n_cells))) return fail(rc);
  if ((rc = h->alloc(&h->d_status, 1))) return fail(rc);
  s.st = h->d_status;
  if (cudaMallocHost((void**)&h->h_status, sizeof(DevStatus)) != cudaSuccess) return fail(GGRID_ENOMEM);
  memset(h->h_status, 0, sizeof(DevStatus));
  if (cudaHostGetDevicePointer((void**)&h->h_status_dev, h->h_status, 0) != cudaSuccess)
    return fail(GGRID_ECUDA);
  h->stats.arena_capacity = cap;
  if (cudaDeviceSynchronize() != cudaSuccess) return fail(GGRID_ECUDA);
  *out = h;
  return GGRID_OK;
}

extern "C" {

int ggrid_free(ggrid_t h) {
  if (!h) return GGRID_OK;
  if (h->multi) {
    multi_free(h->multi);
    delete h;
    return GGRID_OK;
  }
  if (h->xchg) exchange_free(h->xchg);
  for (DBuf& b : h->mx) b.release();
  if (h->stream) cudaStreamSynchronize(h->stream);
  if (h->copy_stream) cudaStreamSynchronize(h->copy_stream);
  for (void* p : h->allocs) cudaFree(p);
  for (DBuf* b : {&h->upd_stage, &h->tmp, &h->q_stage, &h->out_stage, &h->lists, &h->l2_scratch,
                  &h->dump_stage, &h->gc_buf, &h->misc, &h->flush_spill, &h->bound_stage,
                  &h->remote_stage, &h->merge_stage, &h->staged[0].buf,
                  &h->staged[1].buf, &h->qstaged[0].buf, &h->qstaged[1].buf, &h->chain_ring, &h->qsort_buf, &h->resume_buf})
    b->release();
  for (ggrid_s::Staged* sb : {&h->staged[0], &h->staged[1], &h->qstaged[0], &h->qstaged[1]}) {
    if (sb->done) cudaEventDestroy(sb->done);
    if (sb->consumed) cudaEventDestroy(sb->consumed);
  }
  if (h->copy_stream) cudaStreamDestroy(h->copy_stream);
  if (h->ev_in) cudaEventDestroy(h->ev_in);
  if (h->ev_out) cudaEventDestroy(h->ev_out);

  for (auto& pe : h->pending_ev) {
    cudaEventDestroy(pe.second.first);
    cudaEventDestroy(pe.second.second);
  }
  for (cudaEvent_t e : h->ev_pool) cudaEventDestroy(e);
  if (h->h_status) cudaFreeHost(h->h_status);
  if (h->own_stream && h->stream) cudaStreamDestroy(h->stream);
  delete h;
  return GGRID_OK;
}

// (a batch beyond one resident wave over many cells by the sort-by-cell path (1), or always by
// the tile-hash three launches (0))
#ifndef GG_SORTED_INGEST
#define GG_SORTED_INGEST 1
#endif
// ingest n updates already resident in device memory at d_u (the main stream must be
// ordered after their arrival)
static constexpr uint64_t kMaxBatch = 0xFFFFFFFEull;  // seq 2 .. 2^32-1 after a re-base
int ingest_device(ggrid_t h, const uint4* d_u, uint64_t n) {
  if (n > kMaxBatch) return GGRID_EOVERFLOW;
  if (h->async_ingest) RC(h->take_deferred());  // an earlier batch was rejected
  if (h->seq_next + n > 0x100000000ull) RC(h->rebase());
  const uint32_t ext_need = (uint32_t)std::min<uint64_t>(n, h->n_cells);
  RC(h->ensure_arena(n + 3ull * ext_need, ext_need));
  IngestPlan fp;
  const bool fused = h->ingest_mode != 3 && h->ingest_mode != 4 &&
                     ingest_fused_plan(n, h->n_cells, h->sm_count, h->ingest_mode, &fp);
  // beyond one resident wave: the sort-by-cell path (mode 4; by default when the three-launch
  // path's 8,192-update tiles would average under two updates per distinct cell -- C3: 64M-update
  // batch 6.85 -> 6.3 ms; on 264 cells (C1) the tiles aggregate well and the sort loses 3x)
  const bool sorted = !fused && ingest_sorted_fits(n) &&
                      (h->ingest_mode == 4 ||
                       (h->ingest_mode == 0 && GG_SORTED_INGEST && 8192ull <= 2ull * h->n_cells));
  if (!fused) RC(h->tmp.ensure(sorted ? ingest_sort_tmp_bytes(n, h->n_cells) : ingest_tmp_bytes(n)));
  {
    WordSet ws;
    if (fused) ws.add(&h->d_status->ingest_bar, 0u);
    if (h->async_ingest) {  // the previous batch's error bits move to err_deferred (ggrid_sync)
      ws.fold_dst = &h->d_status->err_deferred;
      ws.fold_src = &h->d_status->ingest_err;
    }
    ws.add(&h->d_status->ingest_err, 0u);
    ws.add(&h->d_status->bad_index, 0xFFFFFFFFu);
    ws.add(&h->d_status->batch_tmax, 0u);
    RC(h->set_words(ws));
  }
  const uint32_t seq0 = (uint32_t)h->seq_next;
  const DevGraph& g = h->g;
  const DevState& s = h->s;
  uint2* tmp = h->tmp.as<uint2>();
  cudaStream_t st = h->stream;
  if (fused) {  // one cooperative launch (counted and timed as the classify kind)
    cudaError_t le = cudaSuccess;
    h->launch(GGRID_K_INGEST_CLASSIFY, [&] { le = launch_ingest_fused(d_u, n, seq0, g, s, fp, st); });
    CK(le);
  } else if (sorted) {  // keys + radix sort by cell + runs, extent allocation, sorted scatter
    SortedBatch sb{};
    cudaError_t le = cudaSuccess;
    h->launch(GGRID_K_INGEST_CLASSIFY, [&] { le = launch_ingest_sorted_keys(d_u, n, g, s, h->tmp.p, &sb, st); });
    CK(le);
    h->launch(GGRID_K_INGEST_ALLOC, [&] { launch_ingest_alloc(g, s, st); });
    h->launch(GGRID_K_INGEST_SCATTER, [&] { launch_ingest_sorted_scatter(d_u, n, seq0, g, s, sb, st); });
  } else {
    h->launch(GGRID_K_INGEST_CLASSIFY, [&] { launch_ingest_classify(d_u, n, g, s, tmp, st); });
    h->launch(GGRID_K_INGEST_ALLOC, [&] { launch_ingest_alloc(g, s, st); });
    h->launch(GGRID_K_INGEST_SCATTER, [&] { launch_ingest_scatter(d_u, n, seq0, g, s, tmp, st); });
  }
  if (h->async_ingest) {
    // no host round trip: a rejected batch (checked on the device, all or nothing) keeps its
    // seq range unused, which changes no answer (only the order of keys matters)
    h->pend_records += n + 3ull * ext_need;
    h->pend_ext += ext_need;
    h->pend_updates += n;
    h->seq_next += n;
    h->n_ingested += n;
    h->recs_since_flush += n;
    h->stats.n_updates = h->n_ingested;
    return GGRID_OK;
  }
  RC(h->sync());
  const unsigned err = h->h_status->ingest_err;
  if (err & (ERR_OBJ | ERR_EDGE | ERR_OFF)) {
    if (getenv("GGRID_DEBUG")) {  // diagnosis of a rejected batch (item 0)
      const uint32_t bi = h->h_status->bad_index;
      fprintf(stderr, "ggrid_ingest: batch of %llu rejected, err=0x%x first bad index=%u (%s path)\n",
              (unsigned long long)n, err, bi, fused ? "fused" : "three-launch");
      if (bi < n) {
        uint4 r;
        if (cudaMemcpy(&r, d_u + bi, sizeof(r), cudaMemcpyDeviceToHost) == cudaSuccess)
          fprintf(stderr, "ggrid_ingest: record %u = (obj %u, edge %u, offset %u, t %u)\n", bi, r.x,
                  r.y, r.z, r.w);
      }
    }
    return GGRID_EINVAL;
  }
  if (err & ERR_ARENA) return GGRID_ENOMEM;
  h->seq_next += n;
  h->n_ingested += n;
  h->recs_since_flush += n;
  h->stats.n_updates = h->n_ingested;
  return GGRID_OK;
}

int ggrid_ingest(ggrid_t h, const ggrid_update* u, uint64_t n) {
  if (!h) return GGRID_EINVAL;
  if (n == 0) return GGRID_OK;
  if (!u) return GGRID_EINVAL;
  if (n > kMaxBatch) return GGRID_EOVERFLOW;
  if (h->multi) return multi_ingest(h->multi, u, n);
  CK(cudaSetDevice(h->device));
  const uint4* d_u = reinterpret_cast<const uint4*>(u);
  RC(h->order_inputs(h->stream));  // u may be the output of a caller kernel still running
  if (!is_device_ptr(u)) {
    RC(h->upd_stage.ensure(n * sizeof(uint4)));
    CK(cudaMemcpyAsync(h->upd_stage.p, u, n * sizeof(uint4), cudaMemcpyHostToDevice, h->stream));
    d_u = h->upd_stage.as<uint4>();
  }
  return ingest_device(h, d_u, n);
}

// copy n records of `bytes_each` from src into the next free buffer of a two-deep staging
// ring on the copy stream (the paper's pipelined transfer, P@45017-45625)
static int stage_into(ggrid_t h, ggrid_s::Staged* ring, int head, int count, const void* src, uint64_t n,
                      size_t bytes_each) {
  ggrid_s::Staged& sb = ring[(head + count) & 1];
  if (!sb.done) CK(cudaEventCreateWithFlags(&sb.done, cudaEventDisableTiming));
  if (!sb.consumed) {
    CK(cudaEventCreateWithFlags(&sb.consumed, cudaEventDisableTiming));
    CK(cudaEventRecord(sb.consumed, h->stream));
  }
  sb.n = n;
  // the kernels of this buffer's previous batch may still be reading it
  CK(cudaStreamWaitEvent(h->copy_stream, sb.consumed, 0));
  RC(h->order_inputs(h->copy_stream));  // and src may still be being produced by the caller
  if (n) {
    // both buffers grow together: a cudaMalloc in the middle of a running pipeline stalls it
    RC(ring[0].buf.ensure(n * bytes_each));
    RC(ring[1].buf.ensure(n * bytes_each));
    CK(cudaMemcpyAsync(sb.buf.p, src, n * bytes_each, cudaMemcpyDefault, h->copy_stream));
  }
  CK(cudaEventRecord(sb.done, h->copy_stream));
  return GGRID_OK;
}

int ggrid_ingest_stage(ggrid_t h, const ggrid_update* u, uint64_t n) {
  SINGLE_ONLY(h);
  if (!h || (n && !u) || h->n_staged == 2) return GGRID_EINVAL;
  CK(cudaSetDevice(h->device));
  RC(stage_into(h, h->staged, h->stage_head, h->n_staged, u, n, sizeof(uint4)));
  h->n_staged++;
  return GGRID_OK;
}

int ggrid_query_stage(ggrid_t h, const ggrid_query* q, uint32_t n_q) {
  SINGLE_ONLY(h);
  if (!h || (n_q && !q) || h->n_qstaged == 2) return GGRID_EINVAL;
  CK(cudaSetDevice(h->device));
  RC(stage_into(h, h->qstaged, h->qstage_head, h->n_qstaged, q, n_q, sizeof(uint2)));
  h->n_qstaged++;
  return GGRID_OK;
}

int ggrid_ingest_commit(ggrid_t h) {
  SINGLE_ONLY(h);
  if (!h || h->n_staged == 0) return GGRID_EINVAL;
  CK(cudaSetDevice(h->device));
  ggrid_s::Staged& sb = h->staged[h->stage_head];
  h->stage_head ^= 1;
  h->n_staged--;
  CK(cudaStreamWaitEvent(h->stream, sb.done, 0));
  if (sb.n == 0) return GGRID_OK;
  const int rc = ingest_device(h, sb.buf.as<uint4>(), sb.n);
  CK(cudaEventRecord(sb.consumed, h->stream));
  return rc;
}

#ifndef GG_WIDE_TABLE_HINT
#define GG_WIDE_TABLE_HINT 650.0
#endif
// resumable promotions (knn.cu promote_export): on by default; 0 restarts promoted queries
#ifndef GG_RESUME
#define GG_RESUME 1
#endif
constexpr uint32_t kResumeCap = 4096;  // records per round (~7 KB each at the one-warp level)
#ifndef GG_BALL_FACTOR
#define GG_BALL_FACTOR 2.0  // vertex-table slots per expected ball vertex (experiment hook)
#endif
int knn_impl(ggrid_t h, const ggrid_query* q, uint32_t n_q, uint32_t k, uint32_t* out_obj, uint32_t* out_dist,
             const uint32_t* bound, uint64_t* out_remote) {
  CK(cudaSetDevice(h->device));
  cudaStream_t st = h->stream;
  RC(h->order_inputs(st));  // queries / bounds / outputs may be in use by caller work
  // optional per-query bound (host or device) and remote-rank masks (sharded mode)
  const uint32_t* d_bound = nullptr;
  if (bound) {
    d_bound = static_cast<const uint32_t*>(device_view(bound));
    if (!d_bound) {
      RC(h->bound_stage.ensure((size_t)n_q * 4));
      CK(cudaMemcpyAsync(h->bound_stage.p, bound, (size_t)n_q * 4, cudaMemcpyHostToDevice, st));
      d_bound = h->bound_stage.as<uint32_t>();
    }
  }
  unsigned long long* d_remote = nullptr;
  bool remote_copy = false;
  if (out_remote) {
    d_remote = static_cast<unsigned long long*>(device_view(out_remote));
    if (!d_remote) {
      RC(h->remote_stage.ensure((size_t)n_q * 8));
      d_remote = h->remote_stage.as<unsigned long long>();
      remote_copy = true;
    }
  }
  // every flushed cell writes at most its live objects (+ alignment padding)
  RC(h->ensure_arena(h->flush_need(), 0));
  // device and pinned (mapped) host buffers are used in place — pinned queries and answers
  // cross PCIe inside the kernels and leave the copy engine to a staged ingest batch
  // (ggrid_ingest_stage); pageable host buffers are copied
  const uint2* d_q = static_cast<const uint2*>(device_view(q));
  uint2* q_copy = nullptr;  // pinned queries: the seed kernel copies them into HBM
  if (!d_q) {
    RC(h->q_stage.ensure((size_t)n_q * 8));
    CK(cudaMemcpyAsync(h->q_stage.p, q, (size_t)n_q * 8, cudaMemcpyHostToDevice, st));
    d_q = h->q_stage.as<uint2>();
  } else if (!is_device_ptr(q)) {
    RC(h->q_stage.ensure((size_t)n_q * 8));
    // (not a cudaMemcpyAsync: measured to queue ~170 us behind a staged update batch on the
    // copy engine, while the seed kernel's zero-copy reads take ~50 us under that transfer)
    q_copy = h->q_stage.as<uint2>();
  }
  uint32_t* v_oo = static_cast<uint32_t*>(device_view(out_obj));
  uint32_t* v_od = static_cast<uint32_t*>(device_view(out_dist));
  const bool dev_o = v_oo != nullptr, dev_d = v_od != nullptr;
  uint32_t* d_oo = dev_o ? v_oo : out_obj;
  uint32_t* d_od = dev_d ? v_od : out_dist;
  const size_t outn = (size_t)n_q * k;
  if (!dev_o || !dev_d) {
    RC(h->out_stage.ensure(outn * 8));
    if (!dev_o) d_oo = h->out_stage.as<uint32_t>();
    if (!dev_d) d_od = h->out_stage.as<uint32_t>() + outn;
  }
  const int L = expand_levels();
  RC(h->lists.ensure((size_t)2 * L * n_q * 4));
  uint32_t* lists = h->lists.as<uint32_t>();
  auto list = [&](int buf, int lvl) { return lists + ((size_t)buf * L + lvl) * n_q; };

  h->epoch++;
  const uint32_t epoch = h->epoch;
  // reset err, n_flush, flush_work, n_next[*], flush_end, expand_work[*]
  {
    WordSet ws;
    ws.add(&h->d_status->err, 0u);
    ws.zero_range(&h->d_status->n_flush,
                  (int)((offsetof(DevStatus, round_end) - offsetof(DevStatus, n_flush)) / 4));
    RC(h->set_words(ws));
  }
  const DevGraph& g = h->g;
  const DevState& s = h->s;
  // a batch whose c_q and neighbour cells cover (nearly) every cell requests every dirty cell
  // once instead (flushing a cell no query needs changes no answer: lazy == eager)
  const bool seed_all = h->seed_neighbors && (uint64_t)n_q * (h->max_cell_degree + 1) >= 3ull * h->n_cells;
  const int seed_mode = seed_all ? SEED_ALL : h->seed_neighbors ? SEED_NEIGHBORS : SEED_DST;
  h->launch(GGRID_K_SEED, [&] { launch_seed(d_q, n_q, g, s, epoch, seed_mode, q_copy, st); });
  if (q_copy) d_q = q_copy;

  // starting level: k must fit the candidate list, and the vertex table should hold the
  // expected ball (k objects at the current density need ~k |V| / |O| vertices; the table
  // also holds the frontier and stays below ~1/3 load).  A guess only: a query that
  // overflows is promoted, the answer does not depend on it.
  int lvl0 = 0;
  const double ball = (double)k * h->V / (double)std::max<uint64_t>(1, h->n_live_hi());
  while (lvl0 < L - 2 && (k > expand_max_k(lvl0) || GG_BALL_FACTOR * ball > expand_table_slots(lvl0))) lvl0++;
  while (lvl0 < L - 1 && k > expand_max_k(lvl0)) lvl0++;
  uint32_t ball_hint = (uint32_t)std::min(ball, 1.0e9);  // (bits 30-31: table variant flags)
  if (k > expand_warp_max_k()) ball_hint = std::max(ball_hint, expand_cta_ball());  // (its candidate list)
  // bit 31: the one-warp level 0 takes its wide table (the expected ball touches more vertices:
  // ball x arcs per vertex, C1 ~730 vs C3 ~580)
  if (ball * (double)h->A / std::max(1u, h->V) > GG_WIDE_TABLE_HINT) ball_hint |= 1u << 31;
  else if (k <= 16) ball_hint |= 1u << 30;  // (bit 30: the narrow table's short-candidate-list variant)
  std::vector<uint32_t> n_in(L, 0);
  n_in[lvl0] = n_q;
  // The level above the starting one runs in the same round BESIDE it (a programmatic
  // dependent launch on the same stream, on SM space the starting level leaves free): it takes
  // the queries the starting level promotes as soon as they are written, so a rare overflow
  // costs neither an extra round (a host round trip) nor a serial tail after the starting
  // level.  Deeper promotions wait for the next round.
  const int chain = lvl0 + 1 < L - 1 ? lvl0 + 1 : -1;
  if (chain >= 0) {
    const size_t need = (size_t)n_q * 4;
    if (h->chain_ring.n < need) {
      RC(h->chain_ring.ensure(need));
      CK(cudaMemsetAsync(h->chain_ring.p, 0xFF, h->chain_ring.n, st));  // all NONE
    }
  }
  std::vector<const uint32_t*> in_list(L, nullptr);
  // (experiment hook) the starting level takes the queries in the order of their arcs' source
  // vertices (Z-order ids): spatially close queries run close in time and share L2 lines
  if (getenv("GGRID_SORT_QUERIES") && n_q >= 4096) {
    const size_t tb = sort_queries_tmp_bytes(n_q);
    RC(h->qsort_buf.ensure(tb + (size_t)n_q * 16 + 64));
    unsigned char* base = h->qsort_buf.as<unsigned char>();
    uint32_t* perm = reinterpret_cast<uint32_t*>(base + tb);
    if (launch_sort_queries(d_q, n_q, g, base, tb, perm, st) != 0) return GGRID_ECUDA;
    in_list[lvl0] = perm;
  }
  int cur = 0;
  uint32_t flush_begin = 0;
  for (int round = 0;; ++round) {
    if (round > 100000) return GGRID_ECUDA;
    // round 0 cleans what the seed requested: c_q and its neighbour cells per query
    const uint64_t seeded = seed_all ? h->n_cells : (uint64_t)n_q * (h->seed_neighbors ? h->max_cell_degree + 1 : 2);
    RC(h->flush_list_run(s.ar, &h->d_status->arena_top, flush_begin, 0,
                         round == 0 ? (uint32_t)std::min<uint64_t>(seeded, 1u << 30) : 0, round == 0));
    if (round > 0) {  // round 0 was reset with the rest at the start
      WordSet ws;
      ws.zero_range(h->d_status->n_next, EXPAND_LEVELS);
      ws.zero_range(h->d_status->expand_work, EXPAND_LEVELS);
      ws.add(&h->d_status->n_chain, 0u);
      ws.add(&h->d_status->l0_exited, 0u);
      RC(h->set_words(ws));
    }
    const bool conc = chain >= 0 && n_in[lvl0] > 0;
    // the chained level resumes the starting level's promotions from their exported state
    // (one-warp starting level only; records beyond kResumeCap promote without state)
    uint32_t resume_cap = 0;
    if (conc && GG_RESUME) {
      const size_t rb = expand_resume_bytes(lvl0, n_in[lvl0], h->sm_count, ball_hint);
      if (rb) {
        resume_cap = std::min<uint32_t>(n_in[lvl0], kResumeCap);
        RC(h->resume_buf.ensure(rb * resume_cap));
      }
    }
    const uint32_t grid_c = conc ? std::min<uint32_t>(expand_grid(chain, n_q, h->sm_count, ball_hint), n_in[chain] + 16) : 0;
    uint32_t grid0 = 0;
    if (conc) {  // leave room for the chained level's CTAs (so they are resident from the start)
      const uint32_t full = expand_grid(lvl0, n_in[lvl0], h->sm_count, ball_hint);
      // (in shared memory: a starting-level CTA may hold several queries -- one-warp mode)
      const size_t b0 = expand_block_bytes(lvl0, h->V, n_in[lvl0], h->sm_count, ball_hint, false);
      const size_t bc = expand_block_bytes(chain, h->V, n_q, h->sm_count, ball_hint, true);
      const uint32_t reserve = (uint32_t)((grid_c * bc + b0 - 1) / b0);
      grid0 = full > reserve + h->sm_count ? full - reserve : full;
    }
    auto base = [&](int lvl) {
      ExpandLaunch E;
      E.level = lvl;
      E.q = d_q;
      E.qlist = in_list[lvl];
      E.n = n_in[lvl];
      E.k = k;
      E.epoch = epoch;
      E.retry_list = list(cur ^ 1, lvl);
      E.promote_list = lvl + 1 < L ? list(cur ^ 1, lvl + 1) : nullptr;
      E.promote_count = &h->d_status->n_next[std::min(lvl + 1, L - 1)];
      E.out_obj = d_oo;
      E.out_dist = d_od;
      E.bound = d_bound;
      E.remote = d_remote;
      E.ball_hint = ball_hint;
      if (resume_cap && (lvl == lvl0 || lvl == chain)) {
        E.resume = h->resume_buf.p;
        E.resume_cap = resume_cap;
      }
      return E;
    };
    for (int lvl = 0; lvl < L; ++lvl) {
      if (!n_in[lvl] || (conc && lvl == chain)) continue;
      ExpandLaunch E = base(lvl);
      if (lvl == L - 1) {
        const size_t wb = expand_warp_bytes(lvl, h->V);
        E.scratch_warps = (uint32_t)std::max<size_t>(1, std::min<size_t>(64, (size_t(2) << 30) / wb));
        E.scratch_warps = std::min<uint32_t>(E.scratch_warps, n_in[lvl]);
        RC(h->l2_scratch.ensure(wb * E.scratch_warps));
        E.scratch = h->l2_scratch.p;
      }
      if (conc && lvl == lvl0) {  // promotions go to the chained level running beside
        E.promote_list = h->chain_ring.as<uint32_t>();
        E.promote_count = &h->d_status->n_chain;
        E.exited = &h->d_status->l0_exited;
        E.grid = grid0;
        E.trigger = true;
      }
      const int kind = lvl == 0 ? GGRID_K_EXPAND : GGRID_K_EXPAND_BIG;
      h->launch(kind, [&] {
        launch_expand(E, g, s, h->sm_count, st);
        if (conc && lvl == lvl0) {  // the chained level, started while the starting level runs
          // (inside the same profile-event pair: an event between the two would end the overlap,
          // so in profile mode the pair times the whole expansion phase)
          ExpandLaunch C = base(chain);
          C.chain_in = h->chain_ring.as<uint32_t>();
          C.chain_cap = n_q;
          C.wait_exited = &h->d_status->l0_exited;
          C.wait_total = grid0;
          C.grid = grid_c;
          C.pdl = true;
          h->stats.launches++;
          h->stats.kernel_launches[GGRID_K_EXPAND_BIG]++;
          launch_expand(C, g, s, h->sm_count, st);
        }
      });
    }
    RC(h->sync());
    h->stats.knn_rounds++;
    const unsigned err = h->h_status->err;
    if (err & ERR_QUERY) return GGRID_EINVAL;
    if (err & (ERR_ARENA | ERR_FAIL)) return GGRID_ENOMEM;
    flush_begin = h->h_status->flush_end;
    bool any = false;
    for (int lvl = 0; lvl < L; ++lvl) {
      n_in[lvl] = h->h_status->n_next[lvl];
      in_list[lvl] = list(cur ^ 1, lvl);
      any |= n_in[lvl] != 0;
    }
    cur ^= 1;
    if (!any) break;
  }
  if (!dev_o || !dev_d || remote_copy) {  // (device / pinned outputs were written in place)
    if (!dev_o) CK(cudaMemcpyAsync(out_obj, d_oo, outn * 4, cudaMemcpyDeviceToHost, st));
    if (!dev_d) CK(cudaMemcpyAsync(out_dist, d_od, outn * 4, cudaMemcpyDeviceToHost, st));
    if (remote_copy) CK(cudaMemcpyAsync(out_remote, d_remote, (size_t)n_q * 8, cudaMemcpyDeviceToHost, st));
    RC(h->sync());
  }
  h->stats.n_queries += n_q;
  h->stats.knn_calls++;
  return GGRID_OK;
}

int ggrid_knn_commit(ggrid_t h, uint32_t k, uint32_t* out_obj, uint32_t* out_dist, uint32_t* n_q) {
  SINGLE_ONLY(h);
  if (!h || h->n_qstaged == 0 || k == 0 || k > h->max_k) return GGRID_EINVAL;
  ggrid_s::Staged& sb = h->qstaged[h->qstage_head];
  if (n_q) *n_q = (uint32_t)sb.n;
  if (sb.n && (!out_obj || !out_dist)) return GGRID_EINVAL;
  CK(cudaSetDevice(h->device));
  h->qstage_head ^= 1;
  h->n_qstaged--;
  CK(cudaStreamWaitEvent(h->stream, sb.done, 0));
  int rc = GGRID_OK;
  if (sb.n) rc = knn_impl(h, sb.buf.as<ggrid_query>(), (uint32_t)sb.n, k, out_obj, out_dist);
  CK(cudaEventRecord(sb.consumed, h->stream));
  return rc;
}

int ggrid_knn(ggrid_t h, const ggrid_query* q, uint32_t n_q, uint32_t k, uint32_t* out_obj,
              uint32_t* out_dist) {
  if (!h || k == 0 || k > h->max_k) return GGRID_EINVAL;
  if (h->xchg) {  // one rank of a multi-process index: collective, even with no queries of its own
    if (n_q && (!q || !out_obj || !out_dist)) return GGRID_EINVAL;
    CK(cudaSetDevice(h->device));
    RC(rank_knn(h, q, n_q, k, out_obj, out_dist));
    h->stats.knn_calls++;
    return GGRID_OK;
  }
  if (n_q == 0) return GGRID_OK;
  if (!q || !out_obj || !out_dist) return GGRID_EINVAL;
  if (h->multi) {
    RC(multi_knn(h->multi, q, n_q, k, out_obj, out_dist));
    h->stats.n_queries += n_q;
    h->stats.knn_calls++;
    return GGRID_OK;
  }
  return knn_impl(h, q, n_q, k, out_obj, out_dist);
}

int ggrid_knn_ex(ggrid_t h, const ggrid_query* q, uint32_t n_q, uint32_t k, const uint32_t* bound,
                 uint32_t* out_obj, uint32_t* out_dist, uint64_t* out_remote) {
  SINGLE_ONLY(h);
  if (!h || k == 0 || k > h->max_k) return GGRID_EINVAL;
  if (n_q == 0) return GGRID_OK;
  if (!q || !out_obj || !out_dist) return GGRID_EINVAL;
  return knn_impl(h, q, n_q, k, out_obj, out_dist, bound, out_remote);
}

int ggrid_shard(ggrid_t h, uint32_t n_ranks, uint32_t rank) {
  SINGLE_ONLY(h);
  if (!h || n_ranks == 0 || n_ranks > 64 || rank >= n_ranks || n_ranks > h->n_cells) return GGRID_EINVAL;
  if (h->n_ingested != 0) return GGRID_EINVAL;  // ownership is fixed before the first update
  h->s.n_ranks = n_ranks;
  h->s.rank = rank;
  return GGRID_OK;
}

int ggrid_query_owner(ggrid_t h, const ggrid_query* q, uint32_t n_q, uint32_t* out_rank) {
  SINGLE_ONLY(h);
  if (!h || (n_q && (!q || !out_rank))) return GGRID_EINVAL;
  if (n_q == 0) return GGRID_OK;
  CK(cudaSetDevice(h->device));
  RC(h->order_inputs(h->stream));
  const uint2* d_q = static_cast<const uint2*>(device_view(q));
  if (!d_q) {
    RC(h->q_stage.ensure((size_t)n_q * 8));
    CK(cudaMemcpyAsync(h->q_stage.p, q, (size_t)n_q * 8, cudaMemcpyHostToDevice, h->stream));
    d_q = h->q_stage.as<uint2>();
  }
  uint32_t* d_o = static_cast<uint32_t*>(device_view(out_rank));
  const bool copy = d_o == nullptr;
  if (copy) {
    RC(h->misc.ensure(std::max<size_t>(64, (size_t)n_q * 4)));
    d_o = h->misc.as<uint32_t>();
  }
  h->launch(GGRID_K_OTHER, [&] { launch_query_owner(d_q, n_q, h->g, h->s, d_o, h->stream); });
  if (copy) CK(cudaMemcpyAsync(out_rank, d_o, (size_t)n_q * 4, cudaMemcpyDeviceToHost, h->stream));
  return h->sync();
}

int ggrid_merge_topk(ggrid_t h, uint32_t n_lists, uint32_t n_q, uint32_t k, const uint32_t* lists_obj,
                     const uint32_t* lists_dist, uint32_t* out_obj, uint32_t* out_dist) {
  SINGLE_ONLY(h);
  if (!h || n_lists == 0 || n_lists > 32 || k == 0) return GGRID_EINVAL;
  if (n_q == 0) return GGRID_OK;
  if (!lists_obj || !lists_dist || !out_obj || !out_dist) return GGRID_EINVAL;
  CK(cudaSetDevice(h->device));
  cudaStream_t st = h->stream;
  RC(h->order_inputs(st));
  const size_t in_n = (size_t)n_lists * n_q * k, out_n = (size_t)n_q * k;
  const uint32_t* d_lo = static_cast<const uint32_t*>(device_view(lists_obj));
  const uint32_t* d_ld = static_cast<const uint32_t*>(device_view(lists_dist));
  uint32_t* d_oo = static_cast<uint32_t*>(device_view(out_obj));
  uint32_t* d_od = static_cast<uint32_t*>(device_view(out_dist));
  const bool c_in = !d_lo || !d_ld, c_out = !d_oo || !d_od;
  RC(h->merge_stage.ensure((c_in ? in_n * 8 : 0) + (c_out ? out_n * 8 : 0) + 16));
  uint32_t* sp = h->merge_stage.as<uint32_t>();
  if (c_in) {
    CK(cudaMemcpyAsync(sp, lists_obj, in_n * 4, cudaMemcpyDefault, st));
    CK(cudaMemcpyAsync(sp + in_n, lists_dist, in_n * 4, cudaMemcpyDefault, st));
    d_lo = sp;
    d_ld = sp + in_n;
    sp += 2 * in_n;
  }
  uint32_t* w_o = c_out ? sp : d_oo;
  uint32_t* w_d = c_out ? sp + out_n : d_od;
  h->launch(GGRID_K_OTHER, [&] { launch_merge_topk(n_lists, n_q, k, d_lo, d_ld, w_o, w_d, st); });
  if (c_out) {
    CK(cudaMemcpyAsync(out_obj, w_o, out_n * 4, cudaMemcpyDefault, st));
    CK(cudaMemcpyAsync(out_dist, w_d, out_n * 4, cudaMemcpyDefault, st));
  }
  return h->sync();
}

int ggrid_prior_art_clean(ggrid_t h, uint32_t eta, uint32_t bucket_size, uint32_t write_mode,
                          uint32_t* out_edge, uint32_t* out_off, ggrid_prior_art_result* res) {
  SINGLE_ONLY(h);
  if (!h || (eta != 4 && eta != 5) || bucket_size == 0 || bucket_size > 4096 || write_mode > 1)
    return GGRID_EINVAL;
  CK(cudaSetDevice(h->device));
  cudaStream_t st = h->stream;
  RC(h->sync());
  const uint32_t nc = h->n_cells;
  DBuf cnt, off, scan_tmp, buckets, table, oe, counts;
  auto release = [&] {
    for (DBuf* b : {&cnt, &off, &scan_tmp, &buckets, &table, &oe, &counts}) b->release();
  };
  cudaEvent_t ev[4];
  for (auto& e : ev) CK(cudaEventCreate(&e));
  auto done = [&](int rc) {
    release();
    for (auto& e : ev) cudaEventDestroy(e);
    return rc;
  };
  if (cnt.ensure((size_t)(nc + 1) * 4) || off.ensure((size_t)(nc + 1) * 4) || counts.ensure(16))
    return done(GGRID_ENOMEM);
  const size_t sb = prior_art_scan_bytes(nc + 1);
  if (scan_tmp.ensure(sb)) return done(GGRID_ENOMEM);
  CK(cudaEventRecord(ev[0], st));
  launch_pa_count(h->g, h->s, bucket_size, cnt.as<uint32_t>(), st);
  if (launch_pa_scan(scan_tmp.p, sb, cnt.as<uint32_t>(), off.as<uint32_t>(), nc + 1, st)) return done(GGRID_ECUDA);
  uint32_t n_buckets = 0;
  CK(cudaMemcpyAsync(&n_buckets, off.as<uint32_t>() + nc, 4, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  const uint32_t n_bundles = (n_buckets + (1u << eta) - 1) >> eta;
  const uint64_t tbytes = (uint64_t)h->max_objects * std::max(1u, n_bundles) * 16;
  if (tbytes > (48ull << 30)) return done(GGRID_ENOMEM);
  if (buckets.ensure((size_t)std::max(1u, n_buckets) * prior_art_bucket_bytes()) || table.ensure(tbytes))
    return done(GGRID_ENOMEM);
  launch_pa_fill(h->g, h->s, bucket_size, off.as<uint32_t>(), buckets.p, st);
  CK(cudaMemsetAsync(table.p, 0xFF, tbytes, st));
  CK(cudaMemsetAsync(counts.p, 0, 16, st));
  CK(cudaEventRecord(ev[1], st));
  launch_pa_shuffle(h->s, buckets.p, n_buckets, bucket_size, (int)eta, (int)write_mode, n_bundles, table.p, st);
  CK(cudaEventRecord(ev[2], st));
  uint32_t* d_e = out_edge ? static_cast<uint32_t*>(device_view(out_edge)) : nullptr;
  uint32_t* d_o = out_off ? static_cast<uint32_t*>(device_view(out_off)) : nullptr;
  const bool ce = out_edge && !d_e, co = out_off && !d_o;
  if ((ce || co) && oe.ensure((size_t)h->max_objects * 8)) return done(GGRID_ENOMEM);
  if (ce) d_e = oe.as<uint32_t>();
  if (co) d_o = oe.as<uint32_t>() + h->max_objects;
  launch_pa_collect(h->s, h->max_objects, std::max(1u, n_bundles), table.p, d_e, d_o,
                    counts.as<unsigned long long>(), st);
  CK(cudaEventRecord(ev[3], st));
  unsigned long long hc[2] = {0, 0};
  CK(cudaMemcpyAsync(hc, counts.p, 16, cudaMemcpyDeviceToHost, st));
  if (ce) CK(cudaMemcpyAsync(out_edge, d_e, (size_t)h->max_objects * 4, cudaMemcpyDeviceToHost, st));
  if (co) CK(cudaMemcpyAsync(out_off, d_o, (size_t)h->max_objects * 4, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  CK(cudaGetLastError());
  h->stats.launches += 5;
  if (res) {
    float a = 0, b = 0, c = 0;
    cudaEventElapsedTime(&a, ev[0], ev[1]);
    cudaEventElapsedTime(&b, ev[1], ev[2]);
    cudaEventElapsedTime(&c, ev[2], ev[3]);
    res->ms_prepare = a;
    res->ms_shuffle = b;
    res->ms_collect = c;
    res->n_buckets = n_buckets;
    res->n_bundles = n_bundles;
    res->table_bytes = tbytes;
    res->objects_found = hc[0];
    res->objects_wrong = hc[1];
  }
  return done(GGRID_OK);
}

int ggrid_prior_art_bundle(const uint32_t* obj, const uint64_t* key, uint32_t eta, uint32_t* out_obj,
                           uint64_t* out_key) {
  if (!obj || !key || !out_obj || !out_key || (eta != 4 && eta != 5)) return GGRID_EINVAL;
  const uint32_t n = 1u << eta;
  DBuf b;
  if (b.ensure((size_t)n * 24)) return GGRID_ENOMEM;
  uint32_t* d_o = b.as<uint32_t>();
  unsigned long long* d_k = reinterpret_cast<unsigned long long*>(d_o + 2 * n);
  uint32_t* d_oo = d_o + n;
  unsigned long long* d_ok = d_k + n;
  int rc = GGRID_OK;
  if (cudaMemcpy(d_o, obj, n * 4, cudaMemcpyHostToDevice) || cudaMemcpy(d_k, key, n * 8, cudaMemcpyHostToDevice))
    rc = GGRID_ECUDA;
  if (!rc) {
    launch_pa_bundle(d_o, d_k, (int)eta, d_oo, d_ok, 0);
    if (cudaMemcpy(out_obj, d_oo, n * 4, cudaMemcpyDeviceToHost) ||
        cudaMemcpy(out_key, d_ok, n * 8, cudaMemcpyDeviceToHost))
      rc = GGRID_ECUDA;
  }
  b.release();
  return rc;
}

int ggrid_set_profile(ggrid_t h, uint32_t mask) {
  if (!h) return GGRID_EINVAL;
  if (h->multi) return each_shard(h, [&](ggrid_t x) { return ggrid_set_profile(x, mask); });
  RC(h->sync());  // (collects the events of the previous mode)
  h->profile = mask;
  return GGRID_OK;
}

int ggrid_wait_stream(ggrid_t h, void* stream) {
  if (!h) return GGRID_EINVAL;
  if (h->multi) return each_shard(h, [&](ggrid_t x) { return ggrid_wait_stream(x, stream); });
  CK(cudaSetDevice(h->device));
  cudaStream_t p = static_cast<cudaStream_t>(stream);
  RC(h->order_after(p, h->stream));
  RC(h->order_after(p, h->copy_stream));
  return GGRID_OK;
}

int ggrid_signal_stream(ggrid_t h, void* stream) {
  if (!h) return GGRID_EINVAL;
  if (h->multi) return each_shard(h, [&](ggrid_t x) { return ggrid_signal_stream(x, stream); });
  CK(cudaSetDevice(h->device));
  cudaStream_t c = static_cast<cudaStream_t>(stream);
  if (c == h->stream) return GGRID_OK;
  CK(cudaEventRecord(h->ev_out, h->stream));
  CK(cudaStreamWaitEvent(c, h->ev_out, 0));
  return GGRID_OK;
}

int ggrid_sync(ggrid_t h) {
  if (!h) return GGRID_EINVAL;
  if (h->multi) return each_shard(h, [&](ggrid_t x) { return ggrid_sync(x); });
  CK(cudaSetDevice(h->device));
  RC(h->sync());
  return h->take_deferred();
}

int ggrid_flush_all(ggrid_t h) {
  if (!h) return GGRID_EINVAL;
  if (h->multi) return each_shard(h, [&](ggrid_t x) { return ggrid_flush_all(x); });
  CK(cudaSetDevice(h->device));
  RC(h->ensure_arena(h->flush_need(), 0));
  h->epoch++;
  RC(h->set_status_u32(&h->d_status->n_flush, 0));
  h->launch(GGRID_K_OTHER, [&] { launch_mark_dirty(h->g, h->s, h->epoch, 0, h->stream); });
  RC(h->flush_list_run(h->s.ar, &h->d_status->arena_top, 0));
  RC(h->sync());
  if (h->h_status->err & ERR_ARENA) return GGRID_ENOMEM;
  return GGRID_OK;
}

int ggrid_cell_objects(ggrid_t h, uint32_t cell, uint32_t* obj, uint32_t* edge, uint32_t* off,
                       uint32_t cap, uint32_t* n) {
  if (!h || !n || cell >= h->n_cells) return GGRID_EINVAL;
  if (h->multi)  // the shard owning the cell
    return ggrid_cell_objects(multi_shard(h->multi, (int)owner_of(cell, h->n_cells, multi_n(h->multi))), cell, obj,
                              edge, off, cap, n);
  if (cap && (!obj || !edge || !off)) return GGRID_EINVAL;
  CK(cudaSetDevice(h->device));
  RC(h->ensure_arena(h->flush_need(), 0));
  h->epoch++;
  RC(h->set_status_u32(&h->d_status->n_flush, 1));
  CK(cudaMemcpyAsync(h->s.flush_list, &cell, 4, cudaMemcpyHostToDevice, h->stream));
  RC(h->flush_list_run(h->s.ar, &h->d_status->arena_top, 0));
  RC(h->dump_stage.ensure(16 + (size_t)cap * 12));
  uint32_t* d_n = h->dump_stage.as<uint32_t>();
  uint32_t* d_o = d_n + 4;
  uint32_t* d_e = d_o + cap;
  uint32_t* d_f = d_e + cap;
  RC(h->set_status_u32(d_n, 0));
  h->launch(GGRID_K_OTHER, [&] { launch_dump_cell(h->g, h->s, cell, d_o, d_e, d_f, cap, d_n, h->stream); });
  uint32_t cnt = 0;
  CK(cudaMemcpyAsync(&cnt, d_n, 4, cudaMemcpyDeviceToHost, h->stream));
  RC(h->sync());
  const uint32_t m = std::min(cnt, cap);
  if (m) {
    CK(cudaMemcpy(obj, d_o, (size_t)m * 4, cudaMemcpyDefault));
    CK(cudaMemcpy(edge, d_e, (size_t)m * 4, cudaMemcpyDefault));
    CK(cudaMemcpy(off, d_f, (size_t)m * 4, cudaMemcpyDefault));
  }
  *n = cnt;
  return GGRID_OK;
}

int ggrid_stats(ggrid_t h, ggrid_stats_t* out) {
  if (!h || !out) return GGRID_EINVAL;
  if (h->multi) {  // shard 0's header; work counters and timings summed over the shards
    ggrid_stats_t t{};
    RC(ggrid_stats(multi_shard(h->multi, 0), &t));
    for (uint32_t r = 1; r < multi_n(h->multi); ++r) {
      ggrid_stats_t x{};
      RC(ggrid_stats(multi_shard(h->multi, (int)r), &x));
      t.knn_rounds += x.knn_rounds;
      t.cells_flushed += x.cells_flushed;
      t.records_flushed += x.records_flushed;
      t.objects_written += x.objects_written;
      t.arena_used += x.arena_used;
      t.arena_capacity += x.arena_capacity;
      t.gc_runs += x.gc_runs;
      t.launches += x.launches;
      t.expand_iterations += x.expand_iterations;
      t.expand_vertices += x.expand_vertices;
      t.expand_arcs += x.expand_arcs;
      t.expand_harvested += x.expand_harvested;
      t.expand_objects += x.expand_objects;
      for (int i = 0; i < GGRID_NK; ++i) {
        t.kernel_launches[i] += x.kernel_launches[i];
        t.kernel_ms[i] += x.kernel_ms[i];
      }
      t.records_expired += x.records_expired;
      t.expand_promotions += x.expand_promotions;
      t.expand_retries += x.expand_retries;
      t.remote_requests += x.remote_requests;
      t.expand_resumes += x.expand_resumes;
    }
    t.n_queries = h->stats.n_queries;
    t.knn_calls = h->stats.knn_calls;
    t.n_shards = multi_n(h->multi);
    t.exchange_kind = strcmp(multi_exchange_name(h->multi), "nccl") == 0 ? GGRID_EXCHANGE_NCCL : GGRID_EXCHANGE_LOOPBACK;
    *out = t;
    return GGRID_OK;
  }
  RC(h->sync());
  ggrid_stats_t s = h->stats;
  s.cells_flushed = h->h_status->cells_flushed;
  s.records_flushed = h->h_status->records_flushed;
  s.objects_written = h->h_status->objects_written;
  s.expand_iterations = h->h_status->ex_iters;
  s.expand_vertices = h->h_status->ex_vertices;
  s.expand_arcs = h->h_status->ex_arcs;
  s.expand_harvested = h->h_status->ex_harvested;
  s.expand_objects = h->h_status->ex_objects;
  s.arena_used = h->h_status->arena_top;
  s.arena_capacity = h->s.ar.cap;
  s.n_cells = h->n_cells;
  s.cell_size = h->cs;
  s.delta = h->delta;
  s.n_vertices = h->V;
  s.n_arcs = h->A;
  s.max_objects = h->max_objects;
  s.t_delta = h->t_delta;
  s.t_now = h->h_status->t_max;
  s.records_expired = h->h_status->records_expired;
  s.seq_rebases = h->rebases;
  s.n_shards = h->s.n_ranks;
  s.exchange_kind = h->xchg ? (strcmp(exchange_name(h->xchg), "nccl") == 0 ? GGRID_EXCHANGE_NCCL : 3u) : 0u;
  s.expand_promotions = h->h_status->ex_promoted;
  s.expand_retries = h->h_status->ex_retried;
  s.expand_resumes = h->h_status->ex_resumed;
  *out = s;
  return GGRID_OK;
}

int ggrid_stats_reset(ggrid_t h) {
  if (!h) return GGRID_EINVAL;
  if (h->multi) return each_shard(h, [&](ggrid_t x) { return ggrid_stats_reset(x); });
  RC(h->sync());
  h->stats.launches = 0;
  for (int i = 0; i < GGRID_NK; ++i) {
    h->stats.kernel_launches[i] = 0;
    h->stats.kernel_ms[i] = 0.0;
  }
  return GGRID_OK;
}

int ggrid_vertex_cell(ggrid_t h, uint32_t* cell_of_vertex) {
  if (!h || !cell_of_vertex) return GGRID_EINVAL;
  if (h->multi) return ggrid_vertex_cell(multi_shard(h->multi, 0), cell_of_vertex);
  memcpy(cell_of_vertex, h->user_cell.data(), (size_t)h->V * 4);
  return GGRID_OK;
}

}  // extern "C"

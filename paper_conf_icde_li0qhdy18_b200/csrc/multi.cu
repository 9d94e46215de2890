// multi.cu — one logical index over several shards (include/ggrid.h "multi-GPU").
//
// A shard is an ordinary handle made rank r of R by ggrid_shard: it owns the contiguous
// Z-order range of cells c with floor(c R / n_cells) == r, keeps message logs and cleaned lists
// only for them, and ingests the whole update stream (the object table is replicated, so the
// validity test of reading R8 holds on every shard).  A batch of queries is answered exactly
// with one request/reply exchange (the proof is in ggrid.h, ggrid_shard):
//   route    each query to the owner of its cell                              (all-to-all)
//   primary  owner: its k nearest own objects + the mask of shards whose cells it entered
//   request  (query, bound = owner's k-th distance) to every masked shard      (all-to-all)
//   reply    each such shard: its own objects within the bound, k at most      (all-to-all)
//   merge    owner: first-k of the union (k-way merge kernel, P@51679)
//   return   answers to the shard the query came from                          (all-to-all)
// Every step runs in kernels on the shard's device; the host only sizes buffers (one count
// exchange per variable-size phase) and posts the transfers.  Transports (class Exchange):
//   NcclExchange      ncclSend / ncclRecv in one group per all-to-all (NVLink / NVSwitch);
//                     in-process comms from ncclCommInitAll or one rank's comm from
//                     ncclCommInitRank (multi-process).  libnccl is loaded with dlopen, so the
//                     library has no link-time NCCL dependency (and shares torch's copy).
//   LoopbackExchange  in-process shards (any devices, including several on one device):
//                     peer copies (cudaMemcpyAsync, UVA) between the shards' buffers; lets the
//                     protocol be tested with several shards on one GPU.
//   CallbackExchange  a caller-supplied all-to-all (ggrid_alltoall_fn), e.g. over MPI or
//                     torch.distributed, for multi-process use without NCCL.
#include <dlfcn.h>
#include <nccl.h>

#include <condition_variable>
#include <memory>
#include <mutex>
#include <thread>

#include "handle.cuh"

// ----------------------------------------------------------------------------- transports
struct Exchange {
  virtual ~Exchange() {}
  // Shard r's part of an all-to-all of byte segments: send[p] (sbytes[p]) goes to shard p,
  // recv[p] (rbytes[p], which must equal shard p's sbytes[r]) receives shard p's segment.
  // Device pointers on shard r's device, ordered on stream st.  Returns a GGRID_* code.
  virtual int alltoall(int r, void* const* send, const uint64_t* sbytes, void* const* recv,
                       const uint64_t* rbytes, cudaStream_t st) = 0;
  virtual const char* name() const = 0;
  // An unexpected failure on one shard mid-protocol: release the peers (their pending and
  // later transfers fail instead of waiting forever).  Sticky.
  virtual void abort() {}
};

namespace {

struct Barrier {
  std::mutex m;
  std::condition_variable cv;
  int n = 1, count = 0;
  uint64_t gen = 0;
  bool aborted = false;
  bool wait() {  // false: aborted
    std::unique_lock<std::mutex> lk(m);
    if (aborted) return false;
    const uint64_t g = gen;
    if (++count == n) {
      count = 0;
      ++gen;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return gen != g || aborted; });
    }
    return !aborted;
  }
  void abort() {
    std::lock_guard<std::mutex> lk(m);
    aborted = true;
    cv.notify_all();
  }
};

struct LoopbackExchange : Exchange {
  int n;
  Barrier bar;
  std::vector<void* const*> sends;
  std::vector<const uint64_t*> sb;
  explicit LoopbackExchange(int n_) : n(n_), sends(n_), sb(n_) { bar.n = n_; }
  const char* name() const override { return "loopback"; }
  int alltoall(int r, void* const* send, const uint64_t* sbytes, void* const* recv, const uint64_t* rbytes,
               cudaStream_t st) override {
    // the senders' data must be complete before a peer copies it
    int rc = cudaStreamSynchronize(st) == cudaSuccess ? GGRID_OK : GGRID_ECUDA;
    sends[r] = send;
    sb[r] = sbytes;
    if (!bar.wait()) return GGRID_ECUDA;  // every shard's segments are posted (or a peer failed)
    for (int p = 0; p < n && rc == GGRID_OK; ++p) {
      if (sb[p][r] != rbytes[p]) rc = GGRID_ECUDA;  // (a protocol bug: sizes agree by construction)
      else if (rbytes[p] && cudaMemcpyAsync(recv[p], sends[p][r], rbytes[p], cudaMemcpyDefault, st) != cudaSuccess)
        rc = GGRID_ECUDA;
    }
    if (cudaStreamSynchronize(st) != cudaSuccess) rc = GGRID_ECUDA;
    if (!bar.wait()) return GGRID_ECUDA;  // every copy out of the senders' buffers is done
    return rc;
  }
  void abort() override { bar.abort(); }
};

struct NcclApi {
  ncclResult_t (*getUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*commInitAll)(ncclComm_t*, int, const int*) = nullptr;
  ncclResult_t (*commInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*groupStart)() = nullptr;
  ncclResult_t (*groupEnd)() = nullptr;
  ncclResult_t (*send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*commAbort)(ncclComm_t) = nullptr;
  bool ok = false;
};

const NcclApi& nccl() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    void* so = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!so) so = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!so) return;
    auto sym = [&](const char* n) { return dlsym(so, n); };
    api.getUniqueId = reinterpret_cast<decltype(api.getUniqueId)>(sym("ncclGetUniqueId"));
    api.commInitAll = reinterpret_cast<decltype(api.commInitAll)>(sym("ncclCommInitAll"));
    api.commInitRank = reinterpret_cast<decltype(api.commInitRank)>(sym("ncclCommInitRank"));
    api.commDestroy = reinterpret_cast<decltype(api.commDestroy)>(sym("ncclCommDestroy"));
    api.groupStart = reinterpret_cast<decltype(api.groupStart)>(sym("ncclGroupStart"));
    api.groupEnd = reinterpret_cast<decltype(api.groupEnd)>(sym("ncclGroupEnd"));
    api.send = reinterpret_cast<decltype(api.send)>(sym("ncclSend"));
    api.recv = reinterpret_cast<decltype(api.recv)>(sym("ncclRecv"));
    api.commAbort = reinterpret_cast<decltype(api.commAbort)>(sym("ncclCommAbort"));
    api.ok = api.getUniqueId && api.commInitAll && api.commInitRank && api.commDestroy && api.groupStart &&
             api.groupEnd && api.send && api.recv;
  });
  return api;
}

struct NcclExchange : Exchange {
  std::vector<ncclComm_t> comms;  // comms[r]: shard r's communicator (one entry per process when multi-process)
  int base = 0;                   // the rank of comms[0]
  const char* name() const override { return "nccl"; }
  ~NcclExchange() override {
    for (ncclComm_t c : comms)
      if (c) nccl().commDestroy(c);
  }
  int alltoall(int r, void* const* send, const uint64_t* sbytes, void* const* recv, const uint64_t* rbytes,
               cudaStream_t st) override {
    const NcclApi& a = nccl();
    ncclComm_t c = comms[r - base];
    if (a.groupStart() != ncclSuccess) return GGRID_ENCCL;
    int rc = GGRID_OK;
    for (int p = 0; p < n_ranks; ++p) {
      if (sbytes[p] && a.send(send[p], sbytes[p], ncclUint8, p, c, st) != ncclSuccess) rc = GGRID_ENCCL;
      if (rbytes[p] && a.recv(recv[p], rbytes[p], ncclUint8, p, c, st) != ncclSuccess) rc = GGRID_ENCCL;
    }
    if (a.groupEnd() != ncclSuccess) rc = GGRID_ENCCL;
    return rc;
  }
  void abort() override {
    if (!nccl().commAbort) return;
    for (ncclComm_t& c : comms)
      if (c) {
        nccl().commAbort(c);
        c = nullptr;
      }
  }
  int n_ranks = 1;
};

struct CallbackExchange : Exchange {
  ggrid_alltoall_fn fn;
  void* ctx;
  int n_ranks;
  const char* name() const override { return "callback"; }
  int alltoall(int, void* const* send, const uint64_t* sbytes, void* const* recv, const uint64_t* rbytes,
               cudaStream_t st) override {
    if (cudaStreamSynchronize(st) != cudaSuccess) return GGRID_ECUDA;
    return fn(ctx, send, sbytes, recv, rbytes, (uint32_t)n_ranks, st) == 0 ? GGRID_OK : GGRID_ENCCL;
  }
};

// ----------------------------------------------------------------------------- kernels
// Records exchanged between shards (u32 words):
//   route / request  uint4 {edge, offset, aux, row}   aux = bound (request) or unused (route)
//   reply / answer   k obj, k dist, row               (2k + 1 words)

// per-destination counts of the route phase (dest = owner of the query's cell)
// (an invalid query -- edge >= n_arcs or offset >= w -- sets *err: every shard learns it from the
// count exchange and the whole batch is rejected, EINVAL, on every shard alike)
__global__ void k_route_count(const uint2* __restrict__ q, uint32_t n, DevGraph g, DevState s,
                              uint32_t* __restrict__ dest, uint32_t* __restrict__ counts, uint32_t* __restrict__ err) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint2 qq = q[i];
  uint32_t o = s.rank;
  if (qq.x < g.A) {
    const uint2 ei = g.einfo[qq.x];
    if (qq.y < ei.y) o = owner_of(cellof(g, ei.x), g.n_cells, s.n_ranks);
    else *err = 1u;
  } else {
    *err = 1u;
  }
  dest[i] = o;
  atomicAdd(&counts[o], 1u);
}

// count-exchange records: (count for peer p, this shard's error word)
__global__ void k_count_pairs(const uint32_t* __restrict__ counts, const uint32_t* __restrict__ err, uint32_t R,
                              uint32_t* __restrict__ pairs) {
  const uint32_t p = threadIdx.x;
  if (p < R) {
    pairs[2 * p] = counts[p];
    pairs[2 * p + 1] = *err;
  }
}

// scatter into destination segments (offsets = exclusive scan of counts, computed per CTA from
// the R counts; cursors[R] reset to 0 before)
__global__ void k_route_scatter(const uint2* __restrict__ q, uint32_t n, const uint32_t* __restrict__ dest,
                                const uint32_t* __restrict__ counts, uint32_t R, uint32_t* __restrict__ cursors,
                                uint4* __restrict__ out) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t d = dest[i];
  uint32_t off = 0;
  for (uint32_t p = 0; p < d; ++p) off += counts[p];
  const uint2 qq = q[i];
  out[off + atomicAdd(&cursors[d], 1u)] = make_uint4(qq.x, qq.y, 0u, i);
}

// received route/request records -> the query array (and bounds) a knn call takes
__global__ void k_unpack_queries(const uint4* __restrict__ rec, uint32_t m, uint2* __restrict__ q,
                                 uint32_t* __restrict__ bound) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= m) return;
  const uint4 r = rec[i];
  q[i] = make_uint2(r.x, r.y);
  if (bound) bound[i] = r.z;
}

// requests: one per (row, masked shard) — counts, then scatter
__global__ void k_request_count(const unsigned long long* __restrict__ mask, uint32_t m, uint32_t* __restrict__ counts) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= m) return;
  for (unsigned long long b = mask[i]; b; b &= b - 1) atomicAdd(&counts[__ffsll((long long)b) - 1], 1u);
}
__global__ void k_request_scatter(const uint4* __restrict__ rec, const unsigned long long* __restrict__ mask,
                                  const uint32_t* __restrict__ own_dist, uint32_t m, uint32_t k,
                                  const uint32_t* __restrict__ counts, uint32_t* __restrict__ cursors,
                                  uint4* __restrict__ out) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= m) return;
  const uint32_t bound = own_dist[(size_t)i * k + k - 1];  // the owner's k-th distance (PAD: < k found)
  for (unsigned long long b = mask[i]; b; b &= b - 1) {
    const uint32_t p = __ffsll((long long)b) - 1;
    uint32_t off = 0;
    for (uint32_t j = 0; j < p; ++j) off += counts[j];
    out[off + atomicAdd(&cursors[p], 1u)] = make_uint4(rec[i].x, rec[i].y, bound, i);
  }
}

// (2k+1)-word answer records: row i of (obj, dist) with the row tag taken from rec[i].w
__global__ void k_pack_answers(const uint32_t* __restrict__ obj, const uint32_t* __restrict__ dist,
                               const uint4* __restrict__ rec, uint32_t m, uint32_t k, uint32_t* __restrict__ out) {
  const uint32_t i = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  if (i >= m) return;
  uint32_t* o = out + (size_t)i * (2 * k + 1);
  for (uint32_t j = lane; j < k; j += 32) {
    o[j] = obj[(size_t)i * k + j];
    o[k + j] = dist[(size_t)i * k + j];
  }
  if (lane == 0) o[2 * k] = rec[i].w;
}

// answer records of one source -> rows (row tag) of [slot][rows][k] lists, or of the output
__global__ void k_scatter_answers(const uint32_t* __restrict__ in, uint32_t m, uint32_t k,
                                  uint32_t* __restrict__ obj, uint32_t* __restrict__ dist) {
  const uint32_t i = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  if (i >= m) return;
  const uint32_t* r = in + (size_t)i * (2 * k + 1);
  const size_t row = r[2 * k];
  for (uint32_t j = lane; j < k; j += 32) {
    obj[row * k + j] = r[j];
    dist[row * k + j] = r[k + j];
  }
}

__global__ void k_fill_u32(uint32_t* __restrict__ p, size_t n, uint32_t v) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    p[i] = v;
}

inline uint32_t blocks(uint64_t n, uint32_t per) { return (uint32_t)std::max<uint64_t>(1, (n + per - 1) / per); }

}  // namespace

// ----------------------------------------------------------------------------- one shard's protocol
// Shard r of R answers its origin queries d_q[0..n) (device, on h's device) into d_oo / d_od
// (device, n*k each).  Every shard of the index calls this at the same time (collective).
static int shard_knn(ggrid_t h, Exchange* ex, int r, int R, const uint2* d_q, uint32_t n, uint32_t k,
                     uint32_t* d_oo, uint32_t* d_od) {
  // Any failure from here on leaves the peers inside the protocol: abort the exchange so they
  // fail too instead of waiting (a rejected batch is decided collectively, see k_route_count).
#undef RC
#undef CK
#define RC(x)                  \
  do {                         \
    const int r_ = (x);        \
    if (r_ != GGRID_OK) {      \
      ex->abort();             \
      return r_;               \
    }                          \
  } while (0)
#define CK(x)                                                                  \
  do {                                                                         \
    const cudaError_t e_ = (x);                                                \
    if (e_ != cudaSuccess) {                                                   \
      ex->abort();                                                             \
      return e_ == cudaErrorMemoryAllocation ? GGRID_ENOMEM : GGRID_ECUDA;     \
    }                                                                          \
  } while (0)
  cudaStream_t st = h->stream;
  RC(h->order_inputs(st));
  DBuf* B = h->mx;
  // [0,64) counts, [64,128) cursors, [128,192) count pairs sent, [192,256) pairs received,
  // [256] the error word
  RC(B[0].ensure(4096));
  uint32_t* counts = B[0].as<uint32_t>();
  uint32_t* cursors = counts + 64;
  uint32_t* spairs = counts + 128;
  uint32_t* rpairs = counts + 192;
  uint32_t* err = counts + 256;
  std::vector<uint32_t> sc(R), rcv(R), rq_s(R), rq_r(R);
  auto zero_counts = [&] {
    CK(cudaMemsetAsync(counts, 0, 4 * 128, st));
    return GGRID_OK;
  };
  CK(cudaMemsetAsync(err, 0, 4, st));
  std::vector<void*> sp(R), rp(R);
  std::vector<uint64_t> sbytes(R), rbytes(R);
  std::vector<uint32_t> hp(2 * R), hr(2 * R);
  bool rejected = false;
  // exchange (count for p, error word) pairs -> host copies of sent and received counts
  auto count_exchange = [&](std::vector<uint32_t>& sent, std::vector<uint32_t>& got) {
    k_count_pairs<<<1, 64, 0, st>>>(counts, err, (uint32_t)R, spairs);
    for (int p = 0; p < R; ++p) {
      sp[p] = spairs + 2 * p;
      rp[p] = rpairs + 2 * p;
      sbytes[p] = rbytes[p] = 8;
    }
    RC(ex->alltoall(r, sp.data(), sbytes.data(), rp.data(), rbytes.data(), st));
    CK(cudaMemcpyAsync(hp.data(), spairs, 8 * R, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(hr.data(), rpairs, 8 * R, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    for (int p = 0; p < R; ++p) {
      sent[p] = hp[2 * p];
      got[p] = hr[2 * p];
      rejected |= hr[2 * p + 1] != 0 || hp[2 * p + 1] != 0;
    }
    return GGRID_OK;
  };
  auto data_exchange = [&](void* sbase, const std::vector<uint32_t>& sn, void* rbase, const std::vector<uint32_t>& rn,
                           size_t rec_bytes) {
    size_t so = 0, ro = 0;
    for (int p = 0; p < R; ++p) {
      sp[p] = static_cast<char*>(sbase) + so * rec_bytes;
      rp[p] = static_cast<char*>(rbase) + ro * rec_bytes;
      sbytes[p] = sn[p] * rec_bytes;
      rbytes[p] = rn[p] * rec_bytes;
      so += sn[p];
      ro += rn[p];
    }
    return ex->alltoall(r, sp.data(), sbytes.data(), rp.data(), rbytes.data(), st);
  };
  auto sum = [](const std::vector<uint32_t>& v) {
    uint64_t t = 0;
    for (uint32_t x : v) t += x;
    return t;
  };
  const DevGraph& g = h->g;
  const DevState& s = h->s;

  // ---- route
  RC(zero_counts());
  RC(B[1].ensure((size_t)n * 4 + 16));
  RC(B[2].ensure((size_t)n * 16 + 16));
  if (n) {
    k_route_count<<<blocks(n, 256), 256, 0, st>>>(d_q, n, g, s, B[1].as<uint32_t>(), counts, err);
    k_route_scatter<<<blocks(n, 256), 256, 0, st>>>(d_q, n, B[1].as<uint32_t>(), counts, R, cursors, B[2].as<uint4>());
  }
  h->stats.launches += 2;
  RC(count_exchange(sc, rcv));
  if (rejected) return GGRID_EINVAL;  // (every shard saw the same error words)
  const uint64_t m = sum(rcv);
  RC(B[3].ensure(m * 16 + 16));
  RC(data_exchange(B[2].p, sc, B[3].p, rcv, 16));
  uint4* mine = B[3].as<uint4>();  // grouped by origin shard, in shard order

  // ---- primary: k nearest own objects + the mask of shards entered
  RC(B[4].ensure(m * 8 + 16));   // queries
  RC(B[5].ensure(m * k * 8 + 16));  // own obj + dist
  RC(B[6].ensure(m * 8 + 16));   // masks
  uint2* q_m = B[4].as<uint2>();
  uint32_t* own_o = B[5].as<uint32_t>();
  uint32_t* own_d = own_o + m * k;
  unsigned long long* mask = B[6].as<unsigned long long>();
  if (m) {
    k_unpack_queries<<<blocks(m, 256), 256, 0, st>>>(mine, (uint32_t)m, q_m, nullptr);
    RC(knn_impl(h, reinterpret_cast<const ggrid_query*>(q_m), (uint32_t)m, k, own_o, own_d, nullptr,
                reinterpret_cast<uint64_t*>(mask)));
  }
  // ---- requests to the masked shards
  RC(zero_counts());
  if (m) k_request_count<<<blocks(m, 256), 256, 0, st>>>(mask, (uint32_t)m, counts);
  RC(count_exchange(rq_s, rq_r));
  const uint64_t n_req = sum(rq_s), n_got = sum(rq_r);
  h->stats.remote_requests += n_req;
  RC(B[7].ensure(n_req * 16 + 16));
  RC(B[8].ensure(n_got * 16 + 16));
  if (m && n_req)
    k_request_scatter<<<blocks(m, 256), 256, 0, st>>>(mine, mask, own_d, (uint32_t)m, k, counts, cursors,
                                                      B[7].as<uint4>());
  RC(data_exchange(B[7].p, rq_s, B[8].p, rq_r, 16));
  // ---- replies: own objects within the bound
  const size_t rw = 2 * (size_t)k + 1;  // answer record words
  RC(B[9].ensure(n_got * 12 + n_got * k * 8 + 16));
  RC(B[10].ensure(std::max(n_got, m) * rw * 4 + 16));  // replies sent, then the answers returned
  uint2* got_q = B[9].as<uint2>();
  uint32_t* got_b = reinterpret_cast<uint32_t*>(got_q + n_got);
  uint32_t* rep_o = got_b + n_got;
  uint32_t* rep_d = rep_o + n_got * k;
  uint32_t* rep_rec = B[10].as<uint32_t>();
  if (n_got) {
    k_unpack_queries<<<blocks(n_got, 256), 256, 0, st>>>(B[8].as<uint4>(), (uint32_t)n_got, got_q, got_b);
    RC(knn_impl(h, reinterpret_cast<const ggrid_query*>(got_q), (uint32_t)n_got, k, rep_o, rep_d, got_b, nullptr));
    k_pack_answers<<<blocks(n_got, 8), 256, 0, st>>>(rep_o, rep_d, B[8].as<uint4>(), (uint32_t)n_got, k, rep_rec);
  }
  RC(B[11].ensure(n_req * rw * 4 + 16));
  RC(data_exchange(rep_rec, rq_r, B[11].p, rq_s, rw * 4));  // back to the requesters
  // ---- merge: [R][m][k] lists, own list in slot r, the reply of shard p in slot p
  RC(B[12].ensure((size_t)R * m * k * 8 + 16));
  uint32_t* lo = B[12].as<uint32_t>();
  uint32_t* ld = lo + (size_t)R * m * k;
  uint32_t* fo = B[5].as<uint32_t>();  // (the own lists are copied into slot r first)
  if (m) {
    k_fill_u32<<<std::min<uint64_t>(4096, blocks((uint64_t)R * m * k * 2, 256)), 256, 0, st>>>(lo, (size_t)R * m * k * 2,
                                                                                             GGRID_PAD);
    CK(cudaMemcpyAsync(lo + (size_t)r * m * k, own_o, m * k * 4, cudaMemcpyDeviceToDevice, st));
    CK(cudaMemcpyAsync(ld + (size_t)r * m * k, own_d, m * k * 4, cudaMemcpyDeviceToDevice, st));
    size_t off = 0;
    for (int p = 0; p < R; ++p) {
      if (rq_s[p])
        k_scatter_answers<<<blocks(rq_s[p], 8), 256, 0, st>>>(B[11].as<uint32_t>() + off * rw, rq_s[p], k,
                                                            lo + (size_t)p * m * k, ld + (size_t)p * m * k);
      off += rq_s[p];
    }
    launch_merge_topk((uint32_t)R, (uint32_t)m, k, lo, ld, fo, fo + m * k, st);
    // ---- answers back to the origin shards (route segments reversed)
    k_pack_answers<<<blocks(m, 8), 256, 0, st>>>(fo, fo + m * k, mine, (uint32_t)m, k, rep_rec);
  }
  RC(B[13].ensure((size_t)n * rw * 4 + 16));
  RC(data_exchange(rep_rec, rcv, B[13].p, sc, rw * 4));
  if (n) k_scatter_answers<<<blocks(n, 8), 256, 0, st>>>(B[13].as<uint32_t>(), n, k, d_oo, d_od);
  h->stats.launches += 8;
  CK(cudaStreamSynchronize(st));
  CK(cudaGetLastError());
  return GGRID_OK;
#undef RC
#undef CK
#define RC(x)                      \
  do {                             \
    int r_ = (x);                  \
    if (r_ != GGRID_OK) return r_; \
  } while (0)
#define CK(x)                                                                             \
  do {                                                                                    \
    cudaError_t e_ = (x);                                                                 \
    if (e_ != cudaSuccess) return e_ == cudaErrorMemoryAllocation ? GGRID_ENOMEM : GGRID_ECUDA; \
  } while (0)
}

// ----------------------------------------------------------------------------- the index
struct MultiIndex {
  int n = 0;
  std::vector<ggrid_t> shards;
  std::vector<int> devices;
  std::unique_ptr<Exchange> ex;
  // run fn(r) for every shard concurrently, one host thread per shard (set to its device);
  // returns the first error
  template <class F>
  int run(F&& fn) {
    std::vector<int> rc(n, GGRID_OK);
    std::vector<std::thread> th;
    for (int r = 0; r < n; ++r)
      th.emplace_back([&, r] {
        if (cudaSetDevice(devices[r]) != cudaSuccess) {
          rc[r] = GGRID_ECUDA;
          return;
        }
        rc[r] = fn(r);
      });
    for (auto& t : th) t.join();
    for (int x : rc)
      if (x != GGRID_OK) return x;
    return GGRID_OK;
  }
};

// build-time hooks called by ggrid_build / ggrid_free (api.cu)
int multi_build(const ggrid_graph* gr, uint32_t cell_size, const ggrid_opts& o, ggrid_t* out,
                int (*build_one)(const ggrid_graph*, uint32_t, const ggrid_opts&, ggrid_t*)) {
  const int n = (int)o.n_gpus;
  if (n < 2 || n > 32) return GGRID_EINVAL;
  auto* mi = new (std::nothrow) MultiIndex();
  if (!mi) return GGRID_ENOMEM;
  mi->n = n;
  for (int r = 0; r < n; ++r) mi->devices.push_back(o.devices ? o.devices[r] : r);
  int n_dev = 0;
  if (cudaGetDeviceCount(&n_dev) != cudaSuccess) {
    delete mi;
    return GGRID_ECUDA;
  }
  for (int d : mi->devices)
    if (d < 0 || d >= n_dev) {
      delete mi;
      return GGRID_EINVAL;
    }
  bool distinct = true;
  for (int a = 0; a < n; ++a)
    for (int b = a + 1; b < n; ++b) distinct &= mi->devices[a] != mi->devices[b];
  auto fail = [&](int rc) {
    for (ggrid_t s : mi->shards) ggrid_free(s);
    delete mi;
    return rc;
  };
  const bool want_nccl = o.exchange_kind == GGRID_EXCHANGE_NCCL || (o.exchange_kind == 0 && distinct && nccl().ok);
  if (want_nccl) {
    if (!nccl().ok || !distinct) return fail(GGRID_ENCCL);
    auto* ne = new NcclExchange();
    ne->comms.assign(n, nullptr);
    ne->n_ranks = n;
    mi->ex.reset(ne);
    if (nccl().commInitAll(ne->comms.data(), n, mi->devices.data()) != ncclSuccess) return fail(GGRID_ENCCL);
  } else {
    mi->ex.reset(new LoopbackExchange(n));
  }
  mi->shards.assign(n, nullptr);
  const int rc = mi->run([&](int r) {
    ggrid_opts so = o;
    so.n_gpus = 1;
    so.devices = nullptr;
    so.device = mi->devices[r];
    so.stream = nullptr;  // each shard has its own stream on its device
    int e = build_one(gr, cell_size, so, &mi->shards[r]);
    if (e == GGRID_OK) e = ggrid_shard(mi->shards[r], (uint32_t)n, (uint32_t)r);
    return e;
  });
  if (rc != GGRID_OK) return fail(rc);
  // the front handle: the index's header fields (shard 0's), carrying the shards
  auto* front = new (std::nothrow) ggrid_s();
  if (!front) return fail(GGRID_ENOMEM);
  front->multi = mi;
  front->device = mi->devices[0];
  front->V = mi->shards[0]->V;
  front->A = mi->shards[0]->A;
  front->n_cells = mi->shards[0]->n_cells;
  front->cs = mi->shards[0]->cs;
  front->max_k = mi->shards[0]->max_k;
  front->max_objects = mi->shards[0]->max_objects;
  *out = front;
  return GGRID_OK;
}

void multi_free(MultiIndex* mi) {
  if (!mi) return;
  mi->ex.reset();  // (communicators before the shards' streams)
  for (ggrid_t s : mi->shards) ggrid_free(s);
  delete mi;
}

const char* multi_exchange_name(const MultiIndex* mi) { return mi && mi->ex ? mi->ex->name() : "none"; }
uint32_t multi_n(const MultiIndex* mi) { return mi ? (uint32_t)mi->n : 1u; }
ggrid_t multi_shard(const MultiIndex* mi, int r) { return mi->shards[r]; }

// ingest: every shard ingests the whole batch (replicated object table; appends only own cells)
int multi_ingest(MultiIndex* mi, const ggrid_update* u, uint64_t n) {
  return mi->run([&](int r) { return ggrid_ingest(mi->shards[r], u, n); });
}

// knn: the batch is split into contiguous origin shares (one per shard), answered with the
// exchange protocol, and gathered back into the caller's output rows
int multi_knn(MultiIndex* mi, const ggrid_query* q, uint32_t n_q, uint32_t k, uint32_t* out_obj, uint32_t* out_dist) {
  const int R = mi->n;
  return mi->run([&](int r) {
    ggrid_t h = mi->shards[r];
    const uint32_t base = n_q / R, extra = n_q % R;
    const uint32_t lo = r * base + std::min<uint32_t>(r, extra), cnt = base + (r < (int)extra ? 1 : 0);
    DBuf& in = h->mx[14];
    if (in.ensure((size_t)cnt * 8 + (size_t)cnt * k * 8 + 16) != GGRID_OK ||
        h->order_inputs(h->stream) != GGRID_OK ||
        (cnt && cudaMemcpyAsync(in.p, q + lo, (size_t)cnt * 8, cudaMemcpyDefault, h->stream) != cudaSuccess)) {
      mi->ex->abort();  // (the peers are entering the protocol)
      return GGRID_ENOMEM;
    }
    uint2* d_q = in.as<uint2>();
    uint32_t* d_oo = reinterpret_cast<uint32_t*>(d_q + cnt);
    uint32_t* d_od = d_oo + (size_t)cnt * k;
    RC(shard_knn(h, mi->ex.get(), r, R, d_q, cnt, k, d_oo, d_od));
    if (cnt) {
      CK(cudaMemcpyAsync(out_obj + (size_t)lo * k, d_oo, (size_t)cnt * k * 4, cudaMemcpyDefault, h->stream));
      CK(cudaMemcpyAsync(out_dist + (size_t)lo * k, d_od, (size_t)cnt * k * 4, cudaMemcpyDefault, h->stream));
    }
    CK(cudaStreamSynchronize(h->stream));
    h->stats.n_queries += 0;  // (counted by the knn calls of the protocol)
    return GGRID_OK;
  });
}

// a multi-process shard (opts.n_ranks > 1): this process's part of the protocol
int rank_knn(ggrid_t h, const ggrid_query* q, uint32_t n_q, uint32_t k, uint32_t* out_obj, uint32_t* out_dist) {
  Exchange* ex = h->xchg;
  const int R = (int)h->s.n_ranks, r = (int)h->s.rank;
  DBuf& in = h->mx[14];
  if (in.ensure((size_t)n_q * 8 + (size_t)n_q * k * 8 + 16) != GGRID_OK ||
      h->order_inputs(h->stream) != GGRID_OK ||
      (n_q && cudaMemcpyAsync(in.p, q, (size_t)n_q * 8, cudaMemcpyDefault, h->stream) != cudaSuccess)) {
    ex->abort();
    return GGRID_ENOMEM;
  }
  uint2* d_q = in.as<uint2>();
  uint32_t* d_oo = reinterpret_cast<uint32_t*>(d_q + n_q);
  uint32_t* d_od = d_oo + (size_t)n_q * k;
  RC(shard_knn(h, ex, r, R, d_q, n_q, k, d_oo, d_od));
  if (n_q) {
    CK(cudaMemcpyAsync(out_obj, d_oo, (size_t)n_q * k * 4, cudaMemcpyDefault, h->stream));
    CK(cudaMemcpyAsync(out_dist, d_od, (size_t)n_q * k * 4, cudaMemcpyDefault, h->stream));
  }
  CK(cudaStreamSynchronize(h->stream));
  return GGRID_OK;
}

// multi-process: attach the exchange named by the options to a freshly built shard handle
int rank_attach(ggrid_t h, const ggrid_opts& o) {
  if (o.n_ranks < 2 || o.n_ranks > 32 || o.rank >= o.n_ranks) return GGRID_EINVAL;
  RC(ggrid_shard(h, o.n_ranks, o.rank));
  if (o.exchange) {
    auto* ce = new (std::nothrow) CallbackExchange();
    if (!ce) return GGRID_ENOMEM;
    ce->fn = o.exchange;
    ce->ctx = o.exchange_ctx;
    ce->n_ranks = (int)o.n_ranks;
    h->xchg = ce;
    return GGRID_OK;
  }
  if (!o.nccl_id) return GGRID_EINVAL;
  if (!nccl().ok) return GGRID_ENCCL;
  auto* ne = new (std::nothrow) NcclExchange();
  if (!ne) return GGRID_ENOMEM;
  ne->comms.assign(1, nullptr);
  ne->base = (int)o.rank;
  ne->n_ranks = (int)o.n_ranks;
  h->xchg = ne;
  ncclUniqueId id;
  memcpy(&id, o.nccl_id, sizeof(id));
  if (nccl().commInitRank(&ne->comms[0], (int)o.n_ranks, id, (int)o.rank) != ncclSuccess) return GGRID_ENCCL;
  return GGRID_OK;
}

void exchange_free(Exchange* e) { delete e; }
const char* exchange_name(const Exchange* e) { return e ? e->name() : "none"; }

extern "C" int ggrid_nccl_unique_id(void* out) {
  if (!out) return GGRID_EINVAL;
  if (!nccl().ok) return GGRID_ENCCL;
  ncclUniqueId id;
  if (nccl().getUniqueId(&id) != ncclSuccess) return GGRID_ENCCL;
  memcpy(out, &id, sizeof(id));
  return GGRID_OK;
}

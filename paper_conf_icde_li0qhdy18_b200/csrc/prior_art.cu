// prior_art.cu — the paper's own message-cleaning design, built on B200 as a comparison path
// (not used by ggrid_knn).
//
// Alg. 2 steps 2-4 (P@19259-23566) over the message lists of every cell: the lists are cut
// into buckets of `bucket` messages (the paper's delta^b, tuned to 128, P@60611); one thread
// per bucket reads its messages from the last to the first; bundles of 2^eta threads resolve
// same-object messages with the cache-and-shuffle of Alg. 3 (P@24850-30196, in the order of
// the text and Fig. 3: reading R23) and then write each surviving message into the
// intermediate table T[o][bundle] with mu(eta) rounds of "write if newer" (lines 11-13);
// GPU_Collect (P@23216) takes per object the newest message over the bundles.
//
// Differences forced by the hardware/API, not by the comparison:
//   * messages are compared by the (t, seq) key of reading R7 (the paper compares t);
//   * a T entry (key, arena position) is one 16-byte store, so concurrent writers of one
//     round never tear an entry; the round's winner is whichever lane the memory system
//     keeps, exactly the arbitration the paper's loop relies on;
//   * write_mode 1 replaces the mu(eta) rounds by "repeat until no lane of the bundle is
//     newer" — the bound of Theorem 1 does not hold for bundles mixing objects (SURVEY App.
//     A.2, tests/test_prior_art.py), so mode 0 may install an older message; the result
//     counts those objects (objects_wrong) against the object table.
// T has one entry per (object, bundle): max_objects x bundles x 16 B — the reason this design
// cannot be run at USA scale (the comparison tool reports it).
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include "internal.cuh"

namespace gg {
namespace {

constexpr int ETA_MAX = 5;

struct PaBucket {
  uint32_t start, len;
};

// messages of cell c: its extents (newest batch first) and its cleaned list
__global__ void k_pa_count(DevGraph g, DevState s, uint32_t bsize, uint32_t* __restrict__ cnt) {
  const uint32_t c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c > g.n_cells) return;
  if (c == g.n_cells) {  // scan padding
    cnt[c] = 0;
    return;
  }
  uint32_t n = 0;
  for (uint32_t e = s.cell_head[c]; is_extent(e); e = s.x_next[e]) n += (s.x_len[e] + bsize - 1) / bsize;
  n += (s.cell_comp[c].y + bsize - 1) / bsize;
  cnt[c] = n;
}

__global__ void k_pa_fill(DevGraph g, DevState s, uint32_t bsize, const uint32_t* __restrict__ off,
                          PaBucket* __restrict__ out) {
  const uint32_t c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= g.n_cells) return;
  uint32_t o = off[c];
  auto emit = [&](uint32_t st, uint32_t ln) {
    for (uint32_t a = 0; a < ln; a += bsize) out[o++] = PaBucket{st + a, min(bsize, ln - a)};
  };
  for (uint32_t e = s.cell_head[c]; is_extent(e); e = s.x_next[e]) emit(s.x_start[e], s.x_len[e]);
  emit(s.cell_comp[c].x, s.cell_comp[c].y);
}

struct Msg {
  uint32_t o;               // object (NONE: no message)
  uint32_t pos;             // arena position
  unsigned long long key;   // (t << 32 | seq)
};

__device__ __forceinline__ Msg shfl_xor_msg(const Msg& m, int mask, int width) {
  Msg r;
  r.o = __shfl_xor_sync(0xffffffffu, m.o, mask, width);
  r.pos = __shfl_xor_sync(0xffffffffu, m.pos, mask, width);
  r.key = __shfl_xor_sync(0xffffffffu, m.key, mask, width);
  return r;
}

// Alg. 3 lines 5-9 for one lane: look m's object up in the cache; absent -> add; cached one
// older -> replace; otherwise continue with the cached message
__device__ __forceinline__ void cache_step(Msg (&gam)[ETA_MAX + 1], int& ng, Msg& m) {
  if (m.o == NONE) return;
  for (int i = 0; i < ng; ++i) {
    if (gam[i].o == m.o) {
      if (gam[i].key < m.key) gam[i] = m;
      else m = gam[i];
      return;
    }
  }
  gam[ng++] = m;
}

// Step 1 (cache-and-shuffle) of one bundle message set; lanes in bundles of 2^eta
__device__ __forceinline__ Msg x_shuffle(Msg m, int eta) {
  Msg gam[ETA_MAX + 1];
  int ng = 0;
  const int width = 1 << eta;
  cache_step(gam, ng, m);  // "each thread first adds its message to its message cache"
  for (int j = 1; j <= eta; ++j) {
    m = shfl_xor_msg(m, 1 << (eta - j), width);
    cache_step(gam, ng, m);
  }
  return m;
}

__global__ void k_pa_shuffle(DevState s, const PaBucket* __restrict__ bk, uint32_t n_buckets,
                             uint32_t bsize, int eta, int mu, int write_mode, uint32_t n_bundles,
                             ulonglong2* __restrict__ T) {
  const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;  // bucket index
  const uint32_t bundle = tid >> eta;
  const bool has = tid < n_buckets;
  const PaBucket b = has ? bk[tid] : PaBucket{0, 0};
  const unsigned bundle_mask = (eta == 5) ? 0xffffffffu : (0xffffu << ((threadIdx.x & 31) & 16));
  for (int i = (int)bsize - 1; i >= 0; --i) {  // Alg. 3 line 3: from the bucket's last message
    Msg m;
    m.o = NONE;
    m.pos = 0;
    m.key = 0;
    if (has && (uint32_t)i < b.len) {
      m.pos = b.start + i;
      m.o = s.ar.obj[m.pos];
      m.key = s.ar.key[m.pos];
    }
    m = x_shuffle(m, eta);
    // lines 11-13: repeat mu(eta) times: if T[m.o][bundle].t < m.t then T[m.o][bundle] <- m
    for (int r = 0;; ++r) {
      bool wrote = false;
      if (m.o != NONE) {
        ulonglong2* e = T + (size_t)m.o * n_bundles + bundle;
        const ulonglong2 cur = __ldcg(e);  // L2: sees the previous round's stores
        if (cur.y == ~0ull || cur.x < m.key) {
          __stcg(e, make_ulonglong2(m.key, m.pos));  // one 16-byte store: entries never tear
          wrote = true;
        }
      }
      __syncwarp(bundle_mask);
      if (write_mode == 0) {
        if (r + 1 >= mu) break;
      } else if (!__any_sync(bundle_mask, wrote)) {
        break;
      }
    }
  }
}

// GPU_Collect: per object the newest message over its bundles; counted against ot_key
__global__ void k_pa_collect(DevState s, uint32_t max_objects, uint32_t n_bundles,
                             const ulonglong2* __restrict__ T, uint32_t* __restrict__ out_edge,
                             uint32_t* __restrict__ out_off, unsigned long long* __restrict__ counts) {
  const uint32_t o = blockIdx.x * blockDim.x + threadIdx.x;
  bool found = false, wrong = false;
  if (o < max_objects) {
    unsigned long long best = 0, bpos = ~0ull;
    const ulonglong2* row = T + (size_t)o * n_bundles;
    for (uint32_t b = 0; b < n_bundles; ++b) {
      const ulonglong2 e = row[b];
      if (e.y != ~0ull && (bpos == ~0ull || e.x > best)) {
        best = e.x;
        bpos = e.y;
      }
    }
    found = bpos != ~0ull;
    wrong = found && best != s.ot_key[o];
    if (out_edge) out_edge[o] = found ? s.ar.edge[bpos] : GGRID_PAD;
    if (out_off) out_off[o] = found ? s.ar.off[bpos] : GGRID_PAD;
  }
  const unsigned fm = __ballot_sync(0xffffffffu, found), wm = __ballot_sync(0xffffffffu, wrong);
  if ((threadIdx.x & 31) == 0) {
    if (fm) atomicAdd(&counts[0], (unsigned long long)__popc(fm));
    if (wm) atomicAdd(&counts[1], (unsigned long long)__popc(wm));
  }
}

// one bundle, Step 1 only (test hook): lane i holds (obj[i], key[i])
__global__ void k_pa_bundle(const uint32_t* __restrict__ obj, const unsigned long long* __restrict__ key,
                            int eta, uint32_t* __restrict__ out_obj, unsigned long long* __restrict__ out_key) {
  const int lane = threadIdx.x;  // one full warp; lanes >= 2^eta form other (empty) bundles
  const bool in = lane < (1 << eta);
  Msg m;
  m.o = in ? obj[lane] : NONE;
  m.key = in ? key[lane] : 0;
  m.pos = lane;
  m = x_shuffle(m, eta);
  if (in) {
    out_obj[lane] = m.o;
    out_key[lane] = m.key;
  }
}

}  // namespace

int prior_art_mu(int eta) {
  // Eq. (1) under reading S21: smallest i <= 8 with lambda(eta, i) >= 2^eta
  for (int i = 1; i <= 8; ++i) {
    double lam = i * (eta + 1) * eta / 2.0 + i;
    for (int j = 1; j <= i; ++j) lam -= (14 - j) * (j - 1) / 2.0;
    if (lam >= (double)(1 << eta)) return i;
  }
  double lam8 = 8 * (eta + 1) * eta / 2.0 + 8;
  for (int j = 1; j <= 8; ++j) lam8 -= (14 - j) * (j - 1) / 2.0;
  return (int)((1 << eta) - lam8 + 8);
}

size_t prior_art_scan_bytes(uint32_t n) {
  size_t b = 0;
  cub::DeviceScan::ExclusiveSum(nullptr, b, (const uint32_t*)nullptr, (uint32_t*)nullptr, (int)n);
  return b;
}

void launch_pa_count(const DevGraph& g, const DevState& s, uint32_t bsize, uint32_t* cnt, cudaStream_t st) {
  k_pa_count<<<(g.n_cells + 256) / 256, 256, 0, st>>>(g, s, bsize, cnt);
}
int launch_pa_scan(void* tmp, size_t tmp_bytes, const uint32_t* cnt, uint32_t* off, uint32_t n, cudaStream_t st) {
  return cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, cnt, off, (int)n, st) == cudaSuccess ? 0 : -1;
}
void launch_pa_fill(const DevGraph& g, const DevState& s, uint32_t bsize, const uint32_t* off, void* out,
                    cudaStream_t st) {
  k_pa_fill<<<(g.n_cells + 255) / 256, 256, 0, st>>>(g, s, bsize, off, static_cast<PaBucket*>(out));
}
size_t prior_art_bucket_bytes() { return sizeof(PaBucket); }
void launch_pa_shuffle(const DevState& s, const void* bk, uint32_t n_buckets, uint32_t bsize, int eta,
                       int write_mode, uint32_t n_bundles, void* T, cudaStream_t st) {
  const uint32_t threads = n_bundles << eta;
  if (!threads) return;
  k_pa_shuffle<<<(threads + 255) / 256, 256, 0, st>>>(s, static_cast<const PaBucket*>(bk), n_buckets, bsize,
                                                      eta, prior_art_mu(eta), write_mode, n_bundles,
                                                      static_cast<ulonglong2*>(T));
}
void launch_pa_collect(const DevState& s, uint32_t max_objects, uint32_t n_bundles, const void* T,
                       uint32_t* out_edge, uint32_t* out_off, unsigned long long* counts, cudaStream_t st) {
  k_pa_collect<<<(max_objects + 255) / 256, 256, 0, st>>>(s, max_objects, n_bundles,
                                                          static_cast<const ulonglong2*>(T), out_edge,
                                                          out_off, counts);
}
void launch_pa_bundle(const uint32_t* obj, const unsigned long long* key, int eta, uint32_t* out_obj,
                      unsigned long long* out_key, cudaStream_t st) {
  k_pa_bundle<<<1, 32, 0, st>>>(obj, key, eta, out_obj, out_key);
}

}  // namespace gg

namespace gg {
namespace {
__global__ void k_query_keys(const uint2* __restrict__ q, uint32_t n, DevGraph g, uint32_t* __restrict__ key,
                             uint32_t* __restrict__ idx) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t e = q[i].x;
  key[i] = e < g.A ? g.einfo[e].x : 0u;
  idx[i] = i;
}
}  // namespace
// layout of tmp: [cub temp | keys in | keys out | idx in] ; perm = idx out
size_t sort_queries_tmp_bytes(uint32_t n) {
  size_t t = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, t, (const uint32_t*)nullptr, (uint32_t*)nullptr, (const uint32_t*)nullptr,
                                  (uint32_t*)nullptr, (int)n);
  return ((t + 255) & ~size_t(255)) + 3 * (((size_t)n * 4 + 255) & ~size_t(255));
}
int launch_sort_queries(const uint2* q, uint32_t n, const DevGraph& g, void* tmp, size_t tmp_bytes, uint32_t* perm,
                        cudaStream_t st) {
  size_t t = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, t, (const uint32_t*)nullptr, (uint32_t*)nullptr, (const uint32_t*)nullptr,
                                  (uint32_t*)nullptr, (int)n);
  const size_t ta = (t + 255) & ~size_t(255), na = ((size_t)n * 4 + 255) & ~size_t(255);
  unsigned char* b = static_cast<unsigned char*>(tmp);
  uint32_t* kin = reinterpret_cast<uint32_t*>(b + ta);
  uint32_t* kout = reinterpret_cast<uint32_t*>(b + ta + na);
  uint32_t* iin = reinterpret_cast<uint32_t*>(b + ta + 2 * na);
  k_query_keys<<<(n + 255) / 256, 256, 0, st>>>(q, n, g, kin, iin);
  int bits = 1;
  while (bits < 32 && (1ull << bits) < g.V) ++bits;
  return cub::DeviceRadixSort::SortPairs(b, t, kin, kout, iin, perm, (int)n, 0, bits, st) == cudaSuccess ? 0 : 1;
}
}  // namespace gg

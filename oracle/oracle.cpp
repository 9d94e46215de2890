// oracle/oracle.cpp — the CPU oracle for snapshot kNN over moving objects in road networks.
//
// TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
// cpu_baseline / `--impl reference` legs may load, call or execute this library.  The
// product path (paper_conf_icde_li0qhdy18_b200/) never touches it, and this file shares
// no code, header, table or helper with the CUDA path.
//
// What it computes is the plain definition of the answer, written out:
//
//  1. Snapshot (oracle_snapshot).  For each object o with at least one update,
//     latest(o) = the update of o with max (t, seq), seq = global arrival index.
//     Follows the object table "latest locations of all objects" (P@15869-16250), the
//     "newer message replaces" rule of message cleaning (P@22626-22764) and reading S7
//     ((t, seq) breaks equal timestamps) / S8 (out-of-order arrivals resolved by max).
//  2. Seeds (reading S1).  Query q = <e, d> (P@45698) on arc e = u->v of weight w:
//     d == 0 -> D[u] = 0; otherwise D[v] = w - d.
//  3. Distances.  Dijkstra (binary heap) over the whole directed graph (P@7808-8419:
//     directed weighted graph; Def. 1's "network distance (length of the graph shortest
//     path)", P@9686).
//  4. Object distance.  dist(q,o) = min( D[src(e_o)] + d_o  (P@49436: D[m.e.v_s] + m.d),
//                                        e_o == e_q && d_o >= d_q ? d_o - d_q : inf )
//     (the same-arc term is reading S2).
//  5. Answer (Def. 1, P@9206-9761).  Objects with dist >= 2^32-1 are unreachable
//     (reading S18: distances are 4-byte unsigned integers, P@59405; INF = 2^32-1).
//     Sort by (dist, obj) ascending (reading S5; Fig. 1 order P@3313), output the first
//     min(k, count) and pad with 0xFFFFFFFF (reading S6).
//
// Two modes: FULL (the whole Dijkstra, as north_star specifies) and EARLY (stop when
// the popped distance is strictly greater than the current k-th candidate distance;
// exact because every object at an unpopped vertex is strictly farther).
//
// Everything is in 64-bit unsigned arithmetic internally so no intermediate wraps.
#include <algorithm>
#include <atomic>
#include <cstdint>
#include <cstring>
#include <queue>
#include <thread>
#include <utility>
#include <vector>

namespace {

constexpr uint64_t kInf64 = ~0ull;
constexpr uint64_t kUnreachable = 0xFFFFFFFFull;  // dist >= this is "unreachable" (S18)
constexpr uint32_t kPad = 0xFFFFFFFFu;

struct Graph {
  uint32_t n = 0;
  std::vector<uint64_t> ptr;  // out-arc CSR over source vertices
  std::vector<uint32_t> arc;  // user arc ids grouped by source
  const uint32_t* src = nullptr;
  const uint32_t* dst = nullptr;
  const uint32_t* w = nullptr;
  uint32_t n_arcs = 0;
};

bool make_graph(Graph& g, uint32_t n_vertices, uint32_t n_arcs, const uint32_t* src,
                const uint32_t* dst, const uint32_t* w) {
  g.n = n_vertices;
  g.n_arcs = n_arcs;
  g.src = src;
  g.dst = dst;
  g.w = w;
  g.ptr.assign((size_t)n_vertices + 1, 0);
  for (uint32_t a = 0; a < n_arcs; ++a) {
    if (src[a] >= n_vertices || dst[a] >= n_vertices) return false;
    g.ptr[src[a] + 1]++;
  }
  for (uint32_t v = 0; v < n_vertices; ++v) g.ptr[v + 1] += g.ptr[v];
  std::vector<uint64_t> fill(g.ptr.begin(), g.ptr.end() - 1);
  g.arc.resize(n_arcs);
  for (uint32_t a = 0; a < n_arcs; ++a) g.arc[fill[src[a]]++] = a;
  return true;
}

// Steps 2-3: single-source distances from the on-arc location (q_edge, q_off).
// With early_best == nullptr this is the FULL run; otherwise EARLY mode harvests objects
// at popped vertices into the k best and stops once the popped distance exceeds the k-th.
void dijkstra(const Graph& g, uint32_t q_edge, uint32_t q_off, std::vector<uint64_t>& D,
              const std::vector<uint64_t>* obj_ptr, const std::vector<uint32_t>* obj_at,
              const uint32_t* o_id, const uint32_t* o_edge, const uint32_t* o_off, uint32_t k,
              std::vector<std::pair<uint64_t, uint32_t>>* early_best) {
  D.assign(g.n, kInf64);
  using Item = std::pair<uint64_t, uint32_t>;
  std::priority_queue<Item, std::vector<Item>, std::greater<Item>> pq;
  if (q_off == 0) {
    D[g.src[q_edge]] = 0;
    pq.push({0, g.src[q_edge]});
  } else {
    uint64_t d0 = (uint64_t)g.w[q_edge] - q_off;
    D[g.dst[q_edge]] = d0;
    pq.push({d0, g.dst[q_edge]});
  }
  // EARLY mode keeps the k best (dist, obj) in a max-heap.
  std::priority_queue<Item> best;
  if (early_best) {
    for (auto& p : *early_best) {
      best.push(p);
      if (best.size() > k) best.pop();
    }
  }
  while (!pq.empty()) {
    Item it = pq.top();
    pq.pop();
    uint64_t d = it.first;
    uint32_t u = it.second;
    if (d != D[u]) continue;  // stale heap entry
    if (early_best) {
      if (d >= kUnreachable) break;
      if (best.size() == k && d > best.top().first) break;  // every object at u.. is farther
      for (uint64_t i = (*obj_ptr)[u]; i < (*obj_ptr)[u + 1]; ++i) {
        uint32_t j = (*obj_at)[i];
        if (o_edge[j] == q_edge && o_off[j] >= q_off) continue;  // same-arc term is smaller
        uint64_t od = d + o_off[j];
        if (od >= kUnreachable) continue;
        best.push({od, o_id[j]});
        if (best.size() > k) best.pop();
      }
    }
    for (uint64_t i = g.ptr[u]; i < g.ptr[u + 1]; ++i) {
      uint32_t a = g.arc[i];
      uint64_t nd = d + g.w[a];
      if (nd < D[g.dst[a]]) {
        D[g.dst[a]] = nd;
        pq.push({nd, g.dst[a]});
      }
    }
  }
  if (early_best) {
    early_best->clear();
    while (!best.empty()) {
      early_best->push_back(best.top());
      best.pop();
    }
  }
}

}  // namespace

extern "C" {

// Step 1.  Apply a batch of n updates (rows of 4 u32: obj, edge, offset, t) whose first
// row has global arrival index seq0 to the snapshot state (in/out arrays of n_obj_cap):
// has[o] != 0 iff o has an update; (t[o], seq[o]) is its latest key; edge/off its location.
// Returns 0, or -1 if an object id is out of range.
int oracle_snapshot(uint64_t n, const uint32_t* upd, uint64_t seq0, uint32_t n_obj_cap,
                    uint8_t* has, uint32_t* edge, uint32_t* off, uint32_t* t, uint64_t* seq) {
  for (uint64_t i = 0; i < n; ++i) {
    const uint32_t* m = upd + 4 * i;
    uint32_t o = m[0];
    if (o >= n_obj_cap) return -1;
    uint64_t s = seq0 + i;
    bool newer = !has[o] || m[3] > t[o] || (m[3] == t[o] && s > seq[o]);
    if (newer) {
      has[o] = 1;
      edge[o] = m[1];
      off[o] = m[2];
      t[o] = m[3];
      seq[o] = s;
    }
  }
  return 0;
}

// Steps 2-3 for one location: D (u64, kInf64 = unreachable) for every vertex.
int oracle_vertex_dist(uint32_t n_vertices, uint32_t n_arcs, const uint32_t* src,
                       const uint32_t* dst, const uint32_t* w, uint32_t q_edge, uint32_t q_off,
                       uint64_t* D_out) {
  Graph g;
  if (!make_graph(g, n_vertices, n_arcs, src, dst, w)) return -1;
  if (q_edge >= n_arcs || q_off >= w[q_edge]) return -1;
  std::vector<uint64_t> D;
  dijkstra(g, q_edge, q_off, D, nullptr, nullptr, nullptr, nullptr, nullptr, 0, nullptr);
  std::memcpy(D_out, D.data(), sizeof(uint64_t) * n_vertices);
  return 0;
}

// Steps 2-5 for n_q queries over n_obj existing objects (o_id[j] at (o_edge[j], o_off[j])).
// mode 0 = FULL, 1 = EARLY.  out_obj / out_dist are n_q*k each.  threads <= 0 -> all cores.
int oracle_knn(uint32_t n_vertices, uint32_t n_arcs, const uint32_t* src, const uint32_t* dst,
               const uint32_t* w, uint32_t n_obj, const uint32_t* o_id, const uint32_t* o_edge,
               const uint32_t* o_off, uint32_t n_q, const uint32_t* q_edge, const uint32_t* q_off,
               uint32_t k, int mode, int threads, uint32_t* out_obj, uint32_t* out_dist) {
  if (k == 0) return -1;
  Graph g;
  if (!make_graph(g, n_vertices, n_arcs, src, dst, w)) return -1;
  for (uint32_t j = 0; j < n_obj; ++j)
    if (o_edge[j] >= n_arcs || o_off[j] >= w[o_edge[j]]) return -1;
  for (uint32_t i = 0; i < n_q; ++i)
    if (q_edge[i] >= n_arcs || q_off[i] >= w[q_edge[i]]) return -1;
  // objects grouped by the source vertex of their arc (EARLY mode harvest)
  std::vector<uint64_t> obj_ptr((size_t)n_vertices + 1, 0);
  std::vector<uint32_t> obj_at(n_obj);
  for (uint32_t j = 0; j < n_obj; ++j) obj_ptr[src[o_edge[j]] + 1]++;
  for (uint32_t v = 0; v < n_vertices; ++v) obj_ptr[v + 1] += obj_ptr[v];
  {
    std::vector<uint64_t> fill(obj_ptr.begin(), obj_ptr.end() - 1);
    for (uint32_t j = 0; j < n_obj; ++j) obj_at[fill[src[o_edge[j]]]++] = j;
  }
  unsigned nt = threads > 0 ? (unsigned)threads : std::max(1u, std::thread::hardware_concurrency());
  nt = std::min<unsigned>(nt, std::max<uint32_t>(1, n_q));
  std::atomic<uint32_t> next{0};
  auto worker = [&]() {
    std::vector<uint64_t> D;
    std::vector<std::pair<uint64_t, uint32_t>> cand;
    for (;;) {
      uint32_t qi = next.fetch_add(1);
      if (qi >= n_q) break;
      uint32_t qe = q_edge[qi], qo = q_off[qi];
      cand.clear();
      if (mode == 0) {
        dijkstra(g, qe, qo, D, nullptr, nullptr, nullptr, nullptr, nullptr, 0, nullptr);
        for (uint32_t j = 0; j < n_obj; ++j) {
          uint64_t du = D[src[o_edge[j]]];
          uint64_t d1 = du == kInf64 ? kInf64 : du + o_off[j];
          uint64_t d2 = (o_edge[j] == qe && o_off[j] >= qo) ? (uint64_t)(o_off[j] - qo) : kInf64;
          uint64_t d = std::min(d1, d2);
          if (d < kUnreachable) cand.push_back({d, o_id[j]});
        }
      } else {
        // same-arc objects ahead of q first (their same-arc term is never beaten, S2)
        for (uint64_t i = obj_ptr[src[qe]]; i < obj_ptr[src[qe] + 1]; ++i) {
          uint32_t j = obj_at[i];
          if (o_edge[j] == qe && o_off[j] >= qo) cand.push_back({(uint64_t)(o_off[j] - qo), o_id[j]});
        }
        dijkstra(g, qe, qo, D, &obj_ptr, &obj_at, o_id, o_edge, o_off, k, &cand);
      }
      std::sort(cand.begin(), cand.end());
      uint32_t m = (uint32_t)std::min<size_t>(k, cand.size());
      for (uint32_t r = 0; r < k; ++r) {
        out_obj[(uint64_t)qi * k + r] = r < m ? cand[r].second : kPad;
        out_dist[(uint64_t)qi * k + r] = r < m ? (uint32_t)cand[r].first : kPad;
      }
    }
  };
  std::vector<std::thread> pool;
  for (unsigned i = 1; i < nt; ++i) pool.emplace_back(worker);
  worker();
  for (auto& th : pool) th.join();
  return 0;
}

int oracle_hardware_threads(void) { return (int)std::max(1u, std::thread::hardware_concurrency()); }

}  // extern "C"

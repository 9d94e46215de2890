/* ggrid.h — C ABI of the B200-native lazy-update grid index ("G-Grid") for snapshot
 * kNN queries over moving objects in road networks.
 *
 * Paper: C. Li, Y. Gu, J. Qi, J. He, Q. Deng, G. Yu, "A GPU Accelerated Update Efficient
 * Index for kNN Queries in Road Networks", ICDE 2018.  Citations "P@N" are 0-based
 * character offsets into /root/reference/PAPER.md (one line), see SURVEY.md §0.1.
 *
 * Conventions (all calls):
 *  - Plain pointers and sizes; no torch / C++ types.  Every pointer argument named
 *    "host or device" may be either; the library detects which (cudaPointerGetAttributes)
 *    and never retains it after the call returns -- except under opts.async_ingest, where
 *    a device `u` of ggrid_ingest is read by kernels still queued when the call returns:
 *    it must stay valid and unmodified until the next synchronous call (ggrid_sync,
 *    ggrid_knn, ggrid_flush_all, ggrid_stats, ...) or until a stream ordered after the
 *    library by ggrid_signal_stream reaches it.
 *  - Stream order of caller memory.  Device (and pinned host) memory a call reads or writes
 *    may be produced or consumed by caller work that is still queued.  Each call orders its
 *    device work after everything queued so far on the legacy default stream (which itself
 *    follows every blocking stream) -- or, with opts.stream, after that stream.  Producers on
 *    other non-blocking streams must be named with ggrid_wait_stream before the call.
 *  - Return value 0 = GGRID_OK, negative = error (see GGRID_E*); ggrid_strerror() names it.
 *    On an error no observable state changes (ingest rejects the whole batch).
 *  - All integers are unsigned 32-bit unless noted ("4-byte integers", P@59405).
 *    Distances are u32; a location at network distance >= 2^32-1 is unreachable
 *    (reading R18).  GGRID_PAD = 0xFFFFFFFF pads missing answers.
 *  - The handle is bound to one CUDA device; calls are synchronous on return
 *    (the library's stream is drained) and not thread-safe on the same handle.
 */
#ifndef GGRID_H
#define GGRID_H

#include <stdint.h>

#if defined(__GNUC__)
#pragma GCC visibility push(default) /* the library is built with -fvisibility=hidden */
#endif
#ifdef __cplusplus
extern "C" {
#endif

#define GGRID_OK 0
#define GGRID_EINVAL (-1)    /* bad argument (range, null pointer, k, offsets, ...) */
#define GGRID_ENOMEM (-2)    /* device or host allocation failed / log arena exhausted */
#define GGRID_ECUDA (-3)     /* a CUDA runtime error (sticky errors included) */
#define GGRID_ENCCL (-4)     /* the multi-GPU exchange failed (NCCL or the caller's all-to-all) */
#define GGRID_EOVERFLOW (-5) /* one ingest batch of more than 2^32-2 updates */
#define GGRID_PAD 0xFFFFFFFFu

/* Road network G = <V, E> (P@7808-8419): a directed graph, arc a = src[a] -> dst[a] with
 * weight w[a] >= 1; an undirected road is two arcs of equal weight (P@8380).
 * The ARC INDEX a (0..n_arcs-1) is the edge id used by updates and queries.
 * x, y (optional, may be NULL) are vertex coordinates used only to lay out the grid
 * cells (P@11972-13692); answers never depend on them. All arrays are host pointers. */
typedef struct ggrid_graph {
  uint32_t n_vertices;
  uint32_t n_arcs;
  const uint32_t* src;
  const uint32_t* dst;
  const uint32_t* w;
  const int32_t* x;
  const int32_t* y;
} ggrid_graph;

/* A caller-supplied all-to-all of byte segments (multi-process use without NCCL, see
 * "multi-GPU"): send[p] (send_bytes[p]) goes to rank p; recv[p] (recv_bytes[p]) receives
 * rank p's segment for this rank.  Device pointers on this rank's device; `stream` (a
 * cudaStream_t) has completed all prior work when the function is called, and the function
 * must return only once recv is complete.  Returns 0 on success. */
typedef int (*ggrid_alltoall_fn)(void* ctx, void* const* send, const uint64_t* send_bytes, void* const* recv,
                                 const uint64_t* recv_bytes, uint32_t n_ranks, void* stream);

/* Build options; pass NULL for defaults (each 0 field also means "default"). */
typedef struct ggrid_opts {
  int device;              /* CUDA device ordinal; -1 or 0 = current device       */
  uint32_t max_k;          /* largest k accepted by ggrid_knn (default 256)       */
  uint32_t max_objects;    /* object ids must be < max_objects (default 2^24)     */
  uint64_t log_capacity;   /* record arena capacity in records (default 2^26)     */
  uint32_t delta;          /* expansion bucket width; 0 = mean arc weight          */
  uint32_t seed_neighbors; /* 0 = default on: flush c_q and its neighbour cells up
                              front (Alg. 4 line 1); 2 = off (c_q only)            */
  uint32_t profile;        /* time kernel launches with CUDA events (kernel_ms):
                              bit 0 = every kind, bit k+1 = kind k (GGRID_K_*) only.
                              Each timed launch costs a few microseconds of device
                              idle time between kernels.                           */
  uint32_t t_delta;        /* message expiry window t_Delta (P@20631-21157, sign
                              corrected, reading R21): at cleaning time a
                              cached extent (one ingest batch's messages for one
                              cell) whose newest t is < t_now - t_delta is dropped
                              unread; t_now = the largest t ingested so far.  Exact
                              iff every object reports at least once per t_delta of
                              arrival-ordered time.  0 = never expire.             */
  void* stream;            /* cudaStream_t to run on, or NULL (library stream)    */
  uint32_t async_ingest;   /* 1 = ggrid_ingest / ggrid_ingest_commit return once
                              the batch's kernels are queued on the stream (no
                              host round trip).  Validation still happens, on the
                              device, and still rejects the whole batch; the error
                              (EINVAL, or ENOMEM) is reported later, by the next
                              ggrid_sync or ggrid_ingest call.  A rejected batch
                              leaves its seq range unused.  Ignored (synchronous)
                              when t_delta != 0.  0 = default, synchronous.         */
  uint32_t ingest_kernels; /* 0 = default: a batch that fits one resident wave
                              (<= 8,192 updates per SM) is ingested by ONE
                              cooperative launch (classify, extent allocation and
                              scatter separated by grid barriers) -- the direct
                              variant (one rank atomic per update, no shared
                              memory) when an SM tile would average under two
                              updates per distinct cell, else the shared-memory
                              cell-hash variant when its hash fits -- and larger
                              batches by three launches.  1 = the cell-hash
                              launch whenever it fits; 2 = the direct launch
                              whenever it fits; 3 = always the three launches;
                              4 = the sort-by-cell path (keys, radix sort by cell,
                              per-cell runs, allocation, coalesced scatter) for
                              every batch.  All produce the same index state.      */
  /* ---- multi-GPU (see "multi-GPU" below).  All 0 = one GPU.            */
  uint32_t n_gpus;         /* > 1: ONE index over n_gpus shards driven by this process,
                              shard r on devices[r] (cell ownership, one request/reply
                              exchange per query batch)                            */
  const int* devices;      /* n_gpus device ordinals (NULL = 0 .. n_gpus-1).  An ordinal
                              may repeat (several shards on one device: the loopback
                              exchange -- a test mode of the same protocol)         */
  uint32_t exchange_kind;  /* GGRID_EXCHANGE_*: 0 = auto (NCCL when the devices are
                              distinct and libnccl loads, else loopback)            */
  uint32_t n_ranks, rank;  /* multi-process (one process per GPU): this handle is shard
                              `rank` of `n_ranks`; every rank builds with the same graph
                              and ingests the same update stream                    */
  const void* nccl_id;     /* multi-process over NCCL: the 128-byte ncclUniqueId made by
                              ggrid_nccl_unique_id on one rank and shared by the caller */
  ggrid_alltoall_fn exchange;
                           /* multi-process without NCCL: the caller's all-to-all of
                              byte segments (device pointers on this rank's device;
                              send[p] goes to rank p, recv[p] receives rank p's
                              send[rank]; the stream's prior work is complete when it
                              is called; return 0 on success)                      */
  void* exchange_ctx;      /* passed to exchange                                    */
} ggrid_opts;

#define GGRID_EXCHANGE_AUTO 0u
#define GGRID_EXCHANGE_LOOPBACK 1u
#define GGRID_EXCHANGE_NCCL 2u

typedef struct ggrid_s* ggrid_t;

/* Location update message m = <o, e, d, t> (P@10382-10606): object o is on arc e at
 * distance d from the arc's source (0 <= d < w[e]) at time t.  16 bytes. */
typedef struct ggrid_update {
  uint32_t obj;
  uint32_t edge;
  uint32_t offset;
  uint32_t t;
} ggrid_update;

/* Query q = <k, e, d> (P@45698): a location (edge, offset), 0 <= offset < w[edge]. */
typedef struct ggrid_query {
  uint32_t edge;
  uint32_t offset;
} ggrid_query;

/* Kernel kinds reported by ggrid_stats. */
enum {
  GGRID_K_INGEST_CLASSIFY = 0,
  GGRID_K_INGEST_ALLOC = 1,
  GGRID_K_INGEST_SCATTER = 2,
  GGRID_K_SEED = 3,
  GGRID_K_FLUSH = 4,
  GGRID_K_EXPAND = 5,
  GGRID_K_EXPAND_BIG = 6,
  GGRID_K_OTHER = 7,
  GGRID_NK = 8
};

typedef struct ggrid_stats_t {
  uint64_t n_updates;        /* updates ingested                                     */
  uint64_t n_queries;        /* queries answered                                     */
  uint64_t knn_calls;
  uint64_t knn_rounds;       /* flush+expand rounds over all knn calls               */
  uint64_t cells_flushed;
  uint64_t records_flushed;  /* cached records read by flushes                       */
  uint64_t objects_written;  /* compacted entries written by flushes                 */
  uint64_t arena_used;       /* records (incl. garbage) in the log arena             */
  uint64_t arena_capacity;
  uint64_t gc_runs;
  uint64_t launches;         /* kernel launches issued by the library, all kinds     */
  uint64_t expand_iterations;/* delta-stepping rounds over all answered queries      */
  uint64_t expand_vertices;  /* vertex expansions (out-arc scans)                    */
  uint64_t expand_arcs;      /* arc relaxations                                      */
  uint64_t expand_harvested; /* settled vertices whose object lists were read        */
  uint64_t expand_objects;   /* object entries read while harvesting                 */
  uint64_t kernel_launches[GGRID_NK];
  double kernel_ms[GGRID_NK];/* summed CUDA-event device time (kinds opts.profile times) */
  uint32_t n_cells;
  uint32_t cell_size;
  uint32_t delta;
  uint32_t n_vertices;
  uint32_t n_arcs;
  uint32_t max_objects;
  uint32_t t_delta;          /* opts.t_delta                                          */
  uint32_t t_now;            /* largest t ingested so far                             */
  uint64_t records_expired;  /* cached records dropped unread by t_delta expiry       */
  uint64_t expand_promotions;/* query runs that overflowed a capacity level (rerun on the next) */
  uint64_t expand_retries;   /* query runs stopped by a cell with cached updates (rerun after its flush) */
  uint64_t seq_rebases;      /* re-bases of the arrival index (every ~2^32 updates)  */
  uint32_t n_shards;         /* shards of the index (1: one GPU)                      */
  uint32_t exchange_kind;    /* GGRID_EXCHANGE_* in use (0: none; 3: the caller's all-to-all) */
  uint64_t remote_requests;  /* bounded requests this shard (all shards: summed) sent to others */
  uint64_t expand_resumes;   /* promoted query runs the next level continued from their exported
                                state instead of restarting (a subset of expand_promotions) */
} ggrid_stats_t;

/* Build the index (graph grid, P@11423-15818; object table P@15869; message lists
 * P@16303-17438).  cell_size = the cell capacity delta^c (P@11972): cells are runs of at
 * most cell_size vertices in Z-order (P@13067-13692) of the quantised coordinates.
 * Errors: EINVAL (n_vertices = 0 or >= 2^32-1, arc endpoint out of range, w = 0,
 * cell_size = 0, null pointers, max_k = 0 > 65536), ENOMEM, ECUDA.
 * Ownership: inputs are copied; *out is owned by the caller until ggrid_free. */
int ggrid_build(const ggrid_graph* g, uint32_t cell_size, const ggrid_opts* opts, ggrid_t* out);

/* Append n updates (Alg. 1, P@18177-19248, lazy: P@17773-17981).  Updates are ordered by
 * arrival: u[i] arrives after every update of earlier calls and after u[0..i).  An object's
 * location is its update with the largest (t, arrival) (readings R7/R8); t needs no
 * order.  Internally the arrival index is a 32-bit seq that is re-based (one garbage
 * collection plus a key rewrite, ggrid_stats.seq_rebases) whenever a batch would run past
 * 2^32 - 1, so a handle accepts an unbounded stream.
 * u: host or device pointer to n records.  Errors: EINVAL (obj >= max_objects,
 * edge >= n_arcs, offset >= w[edge]: the whole batch is rejected), EOVERFLOW (a single batch
 * of more than 2^32 - 2 updates), ENOMEM (log arena full even after garbage collection),
 * ECUDA. */
int ggrid_ingest(ggrid_t h, const ggrid_update* u, uint64_t n);

/* Pipelined ingest (the paper's pipelined transfer, P@45017-45625: the GPU works on one group
 * of messages while the next is being received).  ggrid_ingest_stage starts copying n updates
 * (host or device pointer; pinned host memory makes the copy asynchronous) into one of two
 * device staging buffers on a dedicated copy stream and returns at once.  The caller must
 * leave u untouched until the matching ggrid_ingest_commit returns.  ggrid_ingest_commit
 * ingests the oldest staged batch with the semantics and errors of ggrid_ingest (arrival
 * order = commit order).  A ggrid_knn issued between the two calls does not see the staged
 * batch; its kernels overlap the copy.  Errors: EINVAL (stage with both buffers staged,
 * commit with none staged, null u), ENOMEM, ECUDA. */
int ggrid_ingest_stage(ggrid_t h, const ggrid_update* u, uint64_t n);
int ggrid_ingest_commit(ggrid_t h);

/* Pipelined queries, the same two-deep staging for query batches: ggrid_query_stage starts
 * copying n_q queries (host or device pointer) into a device staging buffer on the copy
 * stream, behind any batch staged before it, and returns at once (keep q untouched until the
 * matching ggrid_knn_commit returns).  ggrid_knn_commit answers the oldest staged batch with
 * the semantics and errors of ggrid_knn, and stores its size in *n_q (nullable).  A staged
 * copy competes with nothing on the device: the seed kernel reads HBM instead of reading
 * pinned host queries across PCIe while a staged update batch saturates the link.
 * Errors: EINVAL (stage with both buffers staged, commit with none staged, k, null outputs),
 * ENOMEM, ECUDA. */
int ggrid_query_stage(ggrid_t h, const ggrid_query* q, uint32_t n_q);
int ggrid_knn_commit(ggrid_t h, uint32_t k, uint32_t* out_obj, uint32_t* out_dist, uint32_t* n_q);

/* Answer n_q kNN queries (Def. 1, P@9206-9761; Alg. 4-6, P@44429-52751) on the snapshot
 * of all updates ingested before the call.  Row i of out_obj / out_dist (n_q*k each,
 * host or device pointers) holds the k nearest objects in ascending (dist, obj) order,
 * padded with GGRID_PAD when fewer than k objects are reachable.  Flushes the cells the
 * queries touch (lazy message cleaning, Alg. 2) as a side effect; answers never depend
 * on what was flushed before.  q: host or device pointer to n_q queries.
 * Errors: EINVAL (k = 0 or k > max_k, bad edge/offset, null pointers), ENOMEM, ECUDA. */
int ggrid_knn(ggrid_t h, const ggrid_query* q, uint32_t n_q, uint32_t k, uint32_t* out_obj,
              uint32_t* out_dist);

/* ---- multi-GPU -------------------------------------------------------------
 *
 * An index over R shards answers exactly what one GPU answers (Def. 1).  Shard r owns the
 * contiguous Z-order range of cells c with floor(c R / n_cells) == r (the graph is replicated;
 * logs and cleaned lists live on the owner; the object table is replicated).  The library runs
 * the whole exchange: ggrid_ingest feeds the batch to every shard; ggrid_knn splits the batch
 * into R contiguous origin shares and answers them with one request/reply round (route to
 * the owner of each query's cell, owner's k nearest own objects + the shards its search
 * entered, bounded requests to those shards, replies, first-k merge, answers back), every step
 * in kernels on the shards' devices, transfers over NCCL (ncclSend/ncclRecv groups over
 * NVLink/NVSwitch), peer copies (loopback) or a caller all-to-all (opts.exchange).
 *   - one process, several GPUs:  opts.n_gpus = R (opts.devices);
 *   - one process per GPU:        opts.n_ranks = R, opts.rank, and opts.nccl_id (or
 *                                 opts.exchange); ggrid_knn is then collective: every rank
 *                                 calls it with its own query batch (sizes may differ) and
 *                                 receives the answers to its own rows.
 * On a multi-GPU handle the staged calls (ggrid_*_stage / _commit), ggrid_knn_ex,
 * ggrid_shard, ggrid_query_owner, ggrid_merge_topk and ggrid_prior_art_clean return EINVAL.
 * Errors: ENCCL (libnccl missing, communicator set-up or a transfer failed). */

/* A fresh ncclUniqueId (128 bytes into out) for opts.nccl_id: made on one rank, shared with
 * the others by the caller.  Errors: EINVAL (null), ENCCL (libnccl.so.2 not loadable). */
int ggrid_nccl_unique_id(void* out);

/* ---- cell-ownership sharding primitives (one shard per handle; the protocol's steps) ------
 *
 * ggrid_shard makes this handle rank `rank` of `n_ranks` (<= 64): it owns the contiguous
 * Z-order range of cells c with floor(c * n_ranks / n_cells) == rank.  Every rank ingests the
 * full update stream (the object table stays replicated, so the validity test of reading R8
 * holds everywhere) but keeps message logs and cleaned lists only for its own cells.  Must be
 * called before the first ingest.  Errors: EINVAL (ranges, or updates already ingested).
 *
 * An exact kNN answer then takes one request/reply exchange (orchestrated by the caller over
 * NCCL; paper_conf_icde_li0qhdy18_b200/dist.py):
 *   1. the owner of the query's cell (ggrid_query_owner) runs ggrid_knn_ex with out_remote:
 *      its k nearest among its own objects, and the mask of ranks whose cells the expansion
 *      entered before it stopped;
 *   2. each masked rank runs ggrid_knn_ex with bound = the owner's k-th distance (PAD if the
 *      owner found fewer than k): its own objects within that radius (inclusive), k at most;
 *   3. ggrid_merge_topk merges the owner's list and the replies.
 * Exactness: every object of the global answer is within the owner's k-th distance l; such
 * an object lies at a vertex the owner's expansion settled (all vertices closer than its
 * stopping radius > l), so its cell's owner is in the mask, and that owner's bounded answer
 * contains it (fewer than k of its own objects precede it). */
int ggrid_shard(ggrid_t h, uint32_t n_ranks, uint32_t rank);

/* Owner rank of each query: the rank owning the cell of the query arc's source vertex (where
 * objects on the query's own arc are indexed).  q, out_rank: host or device. */
int ggrid_query_owner(ggrid_t h, const ggrid_query* q, uint32_t n_q, uint32_t* out_rank);

/* ggrid_knn with two optional arguments (NULL = as ggrid_knn):
 *   bound      n_q u32, host or device: return only objects at distance <= bound[i] (rows
 *              padded with GGRID_PAD beyond), and stop expanding past it;
 *   out_remote n_q u64, host or device: bit r set iff the expansion of query i entered a
 *              cell owned by rank r != this rank (sharded handles; 0 otherwise). */
int ggrid_knn_ex(ggrid_t h, const ggrid_query* q, uint32_t n_q, uint32_t k, const uint32_t* bound,
                 uint32_t* out_obj, uint32_t* out_dist, uint64_t* out_remote);

/* Merge n_lists (<= 32) per-query answer lists, each ascending in (dist, obj) and padded with
 * GGRID_PAD, laid out [n_lists][n_q][k] (lists_obj / lists_dist), into the k smallest
 * (dist, obj) per query (the final first-k of the candidate union, P@49436-49765, P@51679).
 * Lists must be disjoint in objects.  Host or device pointers. */
int ggrid_merge_topk(ggrid_t h, uint32_t n_lists, uint32_t n_q, uint32_t k, const uint32_t* lists_obj,
                     const uint32_t* lists_dist, uint32_t* out_obj, uint32_t* out_dist);

/* ---- prior-art comparison path (not used by ggrid_knn) -------------------
 *
 * The paper's message cleaning (Alg. 2 steps 2-4 with Alg. 3 GPU_X_Shuffle and GPU_Collect,
 * P@19259-30196) run on this GPU over the message lists of every cell (cached extents and
 * cleaned lists), read-only: buckets of bucket_size messages, one thread per bucket, bundles of
 * 2^eta threads (eta 4 or 5) resolving same-object messages by cache-and-shuffle (reading R23),
 * then the intermediate table T[object][bundle] written with mu(eta) rounds of "write if newer"
 * (write_mode 0, as printed) or until no lane is newer (write_mode 1), then per object the
 * newest message over the bundles.  out_edge / out_off (nullable; max_objects entries, host or
 * device) receive each object's collected location (GGRID_PAD if none).  T needs
 * max_objects x ceil(buckets / 2^eta) x 16 bytes; ENOMEM beyond 48 GiB. */
typedef struct ggrid_prior_art_result {
  double ms_prepare;        /* bucket table + T reset (CUDA events)                       */
  double ms_shuffle;        /* Alg. 3 over every bucket                                   */
  double ms_collect;        /* GPU_Collect                                                */
  uint64_t n_buckets;
  uint64_t n_bundles;
  uint64_t table_bytes;     /* T                                                          */
  uint64_t objects_found;   /* objects with a message in the lists                        */
  uint64_t objects_wrong;   /* of those, collected message != the object's newest (key)  */
} ggrid_prior_art_result;
int ggrid_prior_art_clean(ggrid_t h, uint32_t eta, uint32_t bucket_size, uint32_t write_mode,
                          uint32_t* out_edge, uint32_t* out_off, ggrid_prior_art_result* res);

/* Test hook: Step 1 (cache-and-shuffle, reading R23) of Alg. 3 on one bundle of 2^eta lanes
 * holding messages (obj[i], key[i]) (host arrays); out_obj / out_key receive the message each
 * lane holds afterwards. */
int ggrid_prior_art_bundle(const uint32_t* obj, const uint64_t* key, uint32_t eta, uint32_t* out_obj,
                           uint64_t* out_key);

/* Order the library after caller work: every device operation of later calls on h starts
 * only after all work queued on `stream` (a cudaStream_t, or NULL = the legacy default
 * stream) before this call has finished -- e.g. the kernel that produced a device update
 * batch on a non-blocking stream.  Event record + stream wait; no host synchronisation.
 * Errors: EINVAL (null h), ECUDA. */
int ggrid_wait_stream(ggrid_t h, void* stream);

/* The converse: work queued on `stream` after this call starts only after every device
 * operation h has queued so far (e.g. the asynchronous ingest of a device buffer the caller
 * wants to reuse or free).  Errors: EINVAL, ECUDA. */
int ggrid_signal_stream(ggrid_t h, void* stream);

/* The paper's query pipeline (Alg. 4-6, P@44429-52751) as a comparison path (
 * not used by ggrid_knn): every dirty cell cleaned first (Alg. 4 l.2, eagerly); per query on
 * the GPU, candidate cells = c_q, its neighbour cells and further rings until they hold
 * >= rho k objects (rho = rho_x100 / 100, the paper's 1.8 is 180), Bellman-Ford over their
 * vertices (Alg. 5), the k nearest of their objects (GPU_First_k) and the unresolved vertices
 * (Def. 3, D <= l inclusive); then Refine_kNN (Alg. 6) on `threads` CPU threads (0 = all
 * cores): a Dijkstra bounded by l - D[v] from every unresolved vertex, the union with the
 * candidates, per-object minimum, first k.  Answers have ggrid_knn's format and must equal
 * its rows (the method is exact under the readings of DESIGN.md).  q: host or device;
 * out_obj / out_dist: HOST pointers (n_q*k).  res (nullable) receives the phase times and
 * work counters.  Errors: EINVAL (k = 0 or > 4096, rho_x100 < 100, null pointers, a multi-GPU
 * handle), ENOMEM (a query beyond the comparison path's caps: 64 candidate cells, 4,096
 * candidate objects or 8,192 unresolved vertices), ECUDA. */
typedef struct ggrid_prior_art_knn_result {
  double ms_clean;           /* flush of every dirty cell                                 */
  double ms_host_index;      /* host vertex -> objects index for the CPU refine          */
  double ms_gpu;             /* Alg. 4 l.1-9 on the GPU (CUDA events)                    */
  double ms_d2h;             /* candidates + unresolved vertices to the host             */
  double ms_cpu_refine;      /* Alg. 6 on CPU threads                                    */
  uint64_t cells;            /* candidate cells, summed over the queries                 */
  uint64_t vertices;         /* vertices of those cells, summed                           */
  uint64_t bf_iterations;    /* Bellman-Ford sweeps, summed                               */
  uint64_t unresolved;       /* unresolved vertices, summed                               */
  uint64_t refine_settled;   /* vertices settled by the refine Dijkstras                  */
  uint32_t threads;          /* CPU threads used                                          */
  uint32_t pad_;
} ggrid_prior_art_knn_result;
int ggrid_prior_art_knn(ggrid_t h, const ggrid_query* q, uint32_t n_q, uint32_t k, uint32_t rho_x100,
                        uint32_t threads, uint32_t* out_obj, uint32_t* out_dist, ggrid_prior_art_knn_result* res);

/* Drain the handle's stream.  Returns the deferred error of an asynchronous ingest batch
 * (opts.async_ingest) that was rejected since the last report, else GGRID_OK; the error is
 * reported once. */
int ggrid_sync(ggrid_t h);

/* Release every resource of h (NULL is accepted). */
int ggrid_free(ggrid_t h);

/* Static string naming rc. */
const char* ggrid_strerror(int rc);

/* ---- test / bench hooks -------------------------------------------------------- */

/* Change opts.profile (the kinds of kernel launches timed with CUDA events) after build. */
int ggrid_set_profile(ggrid_t h, uint32_t mask);

/* Eager message cleaning of every cell with cached updates (lazy == eager invariant). */
int ggrid_flush_all(ggrid_t h);

/* Dump the objects located in `cell` (flushing it first if it has cached updates):
 * up to cap entries of (obj, edge, offset) into host or device arrays; *n receives the
 * number of objects in the cell (may exceed cap).  Order unspecified.
 * Errors: EINVAL (cell >= n_cells, null n). */
int ggrid_cell_objects(ggrid_t h, uint32_t cell, uint32_t* obj, uint32_t* edge, uint32_t* off,
                       uint32_t cap, uint32_t* n);

/* Counters and per-kernel timings (host pointer). */
int ggrid_stats(ggrid_t h, ggrid_stats_t* s);

/* Reset the per-kernel launch counters and timings in ggrid_stats. */
int ggrid_stats_reset(ggrid_t h);

/* The grid partition: cell_of_vertex[v] for every user vertex id (host pointer,
 * n_vertices entries). */
int ggrid_vertex_cell(ggrid_t h, uint32_t* cell_of_vertex);

/* Z-value of grid position (x, y): bits of y and x interleaved, y above x at every
 * level (P@13347-13521: (3,4) -> 37).  Pure host function. */
uint64_t ggrid_zvalue(uint32_t x, uint32_t y);

/* Library version string. */
const char* ggrid_version(void);

#ifdef __cplusplus
}
#endif
#if defined(__GNUC__)
#pragma GCC visibility pop
#endif

#endif /* GGRID_H */

/*
 * tg.h -- C-ABI of the B200-native TempGraph temporal-path query engine.
 *
 * Paper: "TempGraph: An Efficient Chain-driven Temporal Graph Computing
 * Framework on the GPU" (ASPLOS '25), /root/reference/PAPER.md, cited P:L<line>.
 *
 * Model (§2.1): a temporal graph is a list of edges e = (u, v, t, t')
 * with t' = t + duration, optionally weighted (w).  A path e_1..e_k is legal iff
 * t'_i <= t_{i+1}.  A query from x in the window [t_alpha, t_omega]
 * admits paths with t_alpha <= start(P) and end(P) <= t_omega, i.e. an edge can
 * be used iff t >= t_alpha and t + duration <= t_omega (both ends inclusive).
 *
 * Pipeline (§3.2 and Fig. 6):
 *   tg_graph_create  -- copy + validate the edge list (the input of the
 *                       "Chain-based Temporal Graph Transformer")
 *   tg_build_chains  -- transformation into time-dependent chains (Alg. 1,
 *                       P:L229-264) and shortcut generation (Alg. 2)
 *   tg_query         -- Generate-Activate-Compute execution (Alg. 3)
 *
 * Conventions
 *   - Every call returns tg_status; no C++ exception crosses the ABI.  On error
 *     tg_last_error() returns a thread-local message; output buffers are then
 *     unspecified.
 *   - All integers are unsigned 32-bit: vertex ids < n_vertices, times and
 *     durations with t + duration <= TG_TMAX, weights, edge ids (= input index).
 *   - Pointers may be host or device (CUDA) pointers unless stated otherwise;
 *     the library detects which with cudaPointerGetAttributes.  Input arrays are
 *     copied; the caller keeps ownership of everything it passes in.
 *   - A tg_graph is not thread-safe; distinct handles are independent.
 *   - All device work runs on the CUDA device given at create time.
 */
#ifndef TG_H
#define TG_H

#include <stdint.h>

#if defined(__GNUC__)
#define TG_API __attribute__((visibility("default")))
#else
#define TG_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct tg_graph tg_graph; /* opaque; owned by the caller; free with tg_graph_destroy */
typedef struct tg_comm tg_comm;   /* opaque NCCL communicator wrapper (multi-GPU only) */

typedef enum {
    TG_OK = 0,
    TG_ERR_INVALID = 1, /* bad argument: NULL pointer, duration 0, alpha > omega, bad problem */
    TG_ERR_RANGE = 2,   /* id >= n, t + duration > TG_TMAX, source >= n, SP distance overflow */
    TG_ERR_NOMEM = 3,   /* device or host allocation failed */
    TG_ERR_CUDA = 4,    /* any other CUDA runtime error (message in tg_last_error) */
    TG_ERR_STATE = 5,   /* call out of order (e.g. tg_query before tg_build_chains) */
    TG_ERR_NCCL = 6     /* multi-GPU communicator error */
} tg_status;

/* Problems.  TG_LD is not in the paper: it is the north star's
 * latest-departure problem, read as single-TARGET (reading A5). */
typedef enum {
    TG_EAT = 0,      /* earliest arrival time end(P)                         */
    TG_LD = 1,       /* latest departure from v of a path reaching the target by omega */
    TG_FASTEST = 2,  /* min duration(P) = end(P) - start(P), P:L114 (reading A6)       */
    TG_SHORTEST = 3, /* min dist(P) = sum of w_e, P:L115 / P:L185 (reading A7)         */
    TG_REACH = 4,    /* reachability P(u,v) != {}: out = 1 or 0                */
    TG_LD_SOURCE = 5 /* single-SOURCE latest departure (reading R5): the latest start(P)
                        >= t_alpha of a path from the source reaching v by t_omega      */
} tg_problem;

typedef struct {
    uint32_t t_alpha; /* earliest allowed departure of the first edge (inclusive) */
    uint32_t t_omega; /* latest allowed arrival of the last edge (inclusive)      */
} tg_window;

#define TG_UNREACHED 0xFFFFFFFFu /* value and pred sentinel                                     */
#define TG_TMAX 0x7FFFFFFEu      /* max t + duration; keeps (time << 32 | id) words below 2^63  */

/*
 * tg_graph_create -- copy and validate a temporal edge list.
 *   n_vertices  >= 1.
 *   n_edges     number of edges m (0 allowed; m < 2^32 - 1).
 *   u, v        uint32[m] endpoints, each < n_vertices           (else TG_ERR_RANGE)
 *   t_start     uint32[m] departure times t
 *   duration    uint32[m] lambda = t' - t >= 1                    (else TG_ERR_INVALID, reading A2)
 *               t + duration <= TG_TMAX                            (else TG_ERR_RANGE)
 *   weight      uint32[m] or NULL; NULL means weight = duration (reading A7)
 *   device      CUDA device ordinal on which the graph lives.
 *   out_graph   receives the handle.
 * The edge id of edge i is i; predecessors returned by tg_query are edge ids.
 */
TG_API tg_status tg_graph_create(uint32_t n_vertices, uint64_t n_edges,
                          const uint32_t *u, const uint32_t *v, const uint32_t *t_start,
                          const uint32_t *duration, const uint32_t *weight,
                          int device, tg_graph **out_graph);

/*
 * tg_build_chains -- transform the graph (Alg. 1) into disjoint
 * time-dependent chains (Def. 1) of the transformed DAG whose vertices
 * are departure nodes (v, tau) (reading A11), with hubs per Def. 2 (P:L174,
 * P:L225); generate one shortcut per chain (Alg. 2); build the vertex ->
 * occurrence index that replaces the paper's GPU hash table.  The same
 * is done for the time-mirrored graph used by TG_LD (reading A5) unless option
 * "mirror" is 0, in which case the first TG_LD query builds it.  Idempotent.
 * Runs on the legacy default stream and returns when finished.
 */
TG_API tg_status tg_build_chains(tg_graph *g);

/*
 * tg_query -- n_sources independent single-source queries (a batch; reading A10).
 *   p           problem.
 *   sources     HOST uint32[n_sources], each < n_vertices.  For TG_LD they are
 *               targets (reading A5).
 *   n_sources   >= 1.
 *   w           window, t_alpha <= t_omega (else TG_ERR_INVALID).
 *   out         uint32[n_sources * n_vertices], row r = query sources[r]
 *               (host or device).  EAT: arrival time (source: t_alpha);
 *               LD: latest departure (target: t_omega); FASTEST / SHORTEST:
 *               min duration / distance (source: 0); REACH: 1 or 0;
 *               LD_SOURCE: latest departure from the source (source: t_omega).
 *               Unreached vertices read TG_UNREACHED (REACH: 0).
 *   pred        NULL or uint32[n_sources * n_vertices] (host or device), only
 *               for TG_EAT / TG_LD / TG_REACH (else TG_ERR_INVALID).  TG_REACH with
 *               pred == NULL and option "reach_bits" = 1 runs on the bit-lane engine
 *               (64 sources per u64 word over the departure nodes).
 *               EAT/REACH: the smallest
 *               edge id among valid edges e=(u->v) with EAT(u) <= t_e and
 *               t_e + duration_e = EAT(v); LD: the smallest id among first
 *               edges of latest-departure paths (reading A9).  Source/target
 *               and unreached vertices: TG_UNREACHED.
 *   cuda_stream cudaStream_t to run on (NULL = legacy default stream).  The
 *               call returns when the results are in `out` / `pred`.
 * TG_SHORTEST returns TG_ERR_RANGE when the graph's weights could overflow a
 * uint32 distance (max path length x max weight >= 2^32 - 1).
 */
TG_API tg_status tg_query(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t n_sources,
                   tg_window w, uint32_t *out, uint32_t *pred, void *cuda_stream);

/*
 * tg_query_topk -- top-K nearest neighbours per source (the
 * nearest-neighbour workload of P:L116 / P:L134): for source row r, the K vertices
 * v != sources[r] reached by problem p with the smallest values, ascending by
 * (value, vertex id).
 *   p           TG_EAT, TG_FASTEST or TG_SHORTEST (else TG_ERR_INVALID).
 *   K           >= 1.
 *   out_vertex, out_value  uint32[n_sources * K] (host or device), row r at r * K;
 *               rows with fewer than K reached vertices are padded with
 *               TG_UNREACHED in both arrays.
 * The rows are computed with tg_query (same errors) into temporary device memory.
 */
TG_API tg_status tg_query_topk(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t n_sources, tg_window w,
                               uint32_t K, uint32_t *out_vertex, uint32_t *out_value, void *cuda_stream);

/*
 * tg_query_summary -- closeness-style summary of every source row (f4, all-source
 * batches): out_count[r] = number of vertices v != sources[r] with a value (reached),
 * out_sum[r] = the sum of those values (exact, uint64).  HOST arrays uint64[n_sources].
 *   p           TG_EAT, TG_LD, TG_FASTEST, TG_SHORTEST or TG_LD_SOURCE.
 */
TG_API tg_status tg_query_summary(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t n_sources,
                                  tg_window w, uint64_t *out_count, uint64_t *out_sum, void *cuda_stream);

/*
 * tg_graph_insert_edges -- dynamic temporal graphs (§5.6: batches of
 * edge insertions followed by re-transformation).  Appends k edges
 * (same arrays and validation as tg_graph_create; ids continue at the current edge
 * count).  weight must be non-NULL iff the graph was created with weights.  For a
 * built graph the transformation is redone incrementally: the batch alone is sorted
 * and merged into the kept (u, t, id) order of each direction, then nodes, chains,
 * shortcuts and the occurrence index are regenerated; this needs option "dynamic" = 1
 * before tg_build_chains (else TG_ERR_STATE).  Not for partitioned / relabelled graphs
 * (TG_ERR_STATE).  On a validation error the graph keeps its previous edges.
 */
TG_API tg_status tg_graph_insert_edges(tg_graph *g, uint64_t k, const uint32_t *u, const uint32_t *v,
                                       const uint32_t *t_start, const uint32_t *duration, const uint32_t *weight);

/*
 * tg_graph_create_streamed -- a graph larger than the device memory (
 * P:L342-346 §4.5 "Supporting of Out-of-GPU-Memory Processing").  Same edge arrays and
 * validation as tg_graph_create, but they must be HOST memory and are never resident
 * on the device as a whole: they are validated chunk by chunk and cut into blocks of
 * consecutive departure times holding at most block_edges edges each (a topological
 * order of the transformed DAG; one departure time with more edges forms a block of
 * its own), kept in pinned host memory.  tg_build_chains transforms every block on
 * the device (Alg. 1 / Alg. 2 / occurrence index) and keeps the result in pinned host
 * memory; tg_query (TG_EAT, TG_REACH; else TG_ERR_STATE) streams the blocks in time
 * order through two device slots, copying block b+1 while block b is computed.
 * Results are identical to a device-resident graph's.  tg_graph_info reports
 * n_blocks and host_bytes.  Options other than sub_batch / stats / round_group /
 * shortcuts / walk_min have no effect.
 */
TG_API tg_status tg_graph_create_streamed(uint32_t n_vertices, uint64_t n_edges, const uint32_t *u, const uint32_t *v,
                                          const uint32_t *t_start, const uint32_t *duration, const uint32_t *weight,
                                          int device, uint64_t block_edges, tg_graph **out_graph);

TG_API void tg_graph_destroy(tg_graph *g); /* NULL-safe */

TG_API const char *tg_status_string(tg_status s);
TG_API const char *tg_last_error(void); /* thread-local detail of the last error ("" if none) */

/* ---------------------------------------------------------------- introspection */
typedef struct {
    uint32_t n_vertices;
    uint64_t n_edges;
    uint64_t n_nodes;        /* departure nodes N_X = distinct (u, t)                      */
    uint64_t n_chains;       /* time-dependent chains (forward graph)                       */
    uint64_t n_long_chains;  /* chains with >= 2 edges (they carry a computed shortcut)     */
    uint32_t max_chain_len;
    uint32_t c_mirror;       /* C = max(t + duration), the LD mirror constant (reading A5)  */
    uint64_t device_bytes;   /* bytes of device memory held by the graph                    */
    double build_ms;         /* last tg_build_chains wall time                              */
    int built;
    uint64_t n_chains_mirror; /* chains of the LD mirror graph                              */
    uint64_t host_bytes;      /* streamed graphs: pinned host memory holding the time blocks */
    uint32_t n_blocks;        /* streamed graphs: time blocks (0 = device-resident graph)    */
} tg_info;

TG_API tg_status tg_graph_info(const tg_graph *g, tg_info *info);

/*
 * tg_export_chains -- copy the forward chain structure to HOST arrays (tests).
 *   chain_off   uint64[n_chains + 1]: chain c is slots [chain_off[c], chain_off[c+1])
 *   chain_edges uint32[n_edges]: edge id at each slot (chain order)
 *   sc_*        uint32/uint64[n_chains] shortcut per chain (Alg. 2): tail vertex,
 *               tail arrival, sum of w (uint64), elapsed = arr_last - t_first.
 *               Any of the sc_* pointers may be NULL.
 *   mirrored    0 = forward graph, 1 = the LD mirror graph.
 */
TG_API tg_status tg_export_chains(const tg_graph *g, int mirrored, uint64_t *chain_off, uint32_t *chain_edges,
                           uint32_t *sc_tail_v, uint32_t *sc_arr, uint64_t *sc_sum_w, uint32_t *sc_elapsed);

typedef struct {
    uint32_t rounds;          /* GAC rounds of the last tg_query (max over sub-batches)     */
    uint32_t sub_batches;
    uint64_t slots_relaxed;   /* relaxations performed (when stats are enabled)              */
    uint64_t kernel_launches; /* kernels launched by the last tg_query                       */
    uint64_t slots_union;     /* distinct slots relaxed by any query of a sub-batch, summed over
                                 sub-batches (stats enabled; EAT/LD): W_union of SURVEY 8(d).
                                 SP/FP/LD_SOURCE: slots_relaxed = chain-slot relaxations,
                                 slots_union = wait-edge steps (node states updated by waiting) */
} tg_query_stats;

/* Statistics of the last tg_query on this handle.  If per_query_relax is not
 * NULL and stats are enabled it receives uint64[n_sources]: slots relaxed per
 * query (equals the one-pass work count W for EAT/LD: each valid usable edge is
 * relaxed exactly once, "first touch"). */
TG_API tg_status tg_last_query_stats(const tg_graph *g, tg_query_stats *st, uint64_t *per_query_relax);

/* ---------------------------------------------------------------- multi-GPU
 * Two ways to use N GPUs; every rank calls the same functions with
 * the same arguments (SPMD), one process per GPU.
 *   mode 0 (replicate): each rank builds a full replica and answers its own block
 *     of sources -- no communication on the data path; nothing to attach.
 *   mode 1 (vertex range): ONE query batch is partitioned: rank r owns vertices
 *     [n*r/N, n*(r+1)/N) and the chains of the edges leaving them (and, for LD,
 *     of the mirror edges leaving them).  After every GAC round the packed
 *     (arrival << 32 | pred) states -- u32 arrivals when pred == NULL -- are combined
 *     with ncclAllReduce(min) over NVLink; `out`/`pred` are complete on every rank.  EAT / LD / REACH only.
 * NCCL is loaded at run time (dlopen "libnccl.so.2"), sharing the process's copy. */

/* 128-byte ncclUniqueId for tg_comm_create (rank 0 creates it, the caller broadcasts it). */
TG_API tg_status tg_nccl_unique_id(void *out_id);
/* Communicator for (rank, world) on `device`; world == 1 needs no NCCL. */
TG_API tg_status tg_comm_create(const void *nccl_unique_id, int rank, int world, int device, tg_comm **out);
TG_API void tg_comm_destroy(tg_comm *c); /* NULL-safe; destroy graphs that use it first */
/* Attach before tg_build_chains; mode 0 = replicate, 1 = vertex range. */
TG_API tg_status tg_graph_attach_comm(tg_graph *g, tg_comm *c, int mode);

/* Tuning / debugging knobs (key, value):
 *   "sub_batch"  sources processed concurrently (0 = automatic)
 *   "stats"      1 = count relaxations per query (slower), 0 = off
 *   "shortcuts"  1 = relax chain tails through shortcuts on first entry (default), 0 = off
 *   "round_group" rounds launched between host convergence checks (default 8)
 *   "mirror"     1 = build the LD mirror in tg_build_chains (default), 0 = on first LD query
 *   "walk_min"   chains with at least this many edges are walked by the chain engine
 *                (default 6, min 2, before build); shorter chains are relaxed edge by
 *                edge through their own occurrences (P:L322's RemoveChain, generalised)
 *   "relabel"    1 = internal vertex order by descending in-degree (before build; default 0:
 *                no gain measured on R-MAT); invisible to callers
 *   "partitions" logical vertex-range partitions on this GPU (1..16, before build):
 *                runs the multi-GPU mode-1 algorithm inside one process (tests)
 *   "exchange"   1 = vertex-range partitions run the cross-rank algorithm even inside one
 *                process: logical partitions relax private state copies that are combined
 *                by an elementwise-min kernel after every round (the stand-in for
 *                ncclAllReduce(min)); a communicator of world 1 calls NCCL itself.  Every
 *                partition then derives its next frontier from the combined state, as
 *                the ranks of a multi-GPU run do (tests; default 0: one process shares
 *                one state and frontier)
 *   "reach_bits" 1 = TG_REACH without pred runs the bit-lane engine: one bit per (departure
 *                node, source), 64 sources per u64 word (8 B per node per 64 sources instead of
 *                4 B of arrival + 4 B of boundary per (vertex, source)); default 0: the EAT
 *                engine, which is faster on the measured configs
 *   "dynamic"    1 = keep each direction's sorted edge order (before build; 4 B per edge
 *                and direction) so tg_graph_insert_edges re-transforms incrementally
 *   "order_sources" 1 (default) = a call's sources are cut into sub-batches in order of
 *                their first departure time >= t_alpha (results still go to the caller's
 *                rows); 0 = in the caller's order
 *   "packed_state" 1 = EAT/LD/REACH keep the packed u64 (arrival << 32 | pred) state even
 *                when pred == NULL (default 0: without pred the state is the u32 arrival
 *                alone -- half the state bytes; values are identical)
 *   "ub_filter"  EAT/LD/REACH batches of 2..64 queries: per (vertex, 8 queries) an 8-bit
 *                code of an upper bound of their arrivals, refreshed at activation, lets
 *                an edge skip the queries it cannot improve before any state read.
 *                0 = off, 1 (default) = on when the sub-batch state is >= 1 GiB, 2 = on.
 *                Results are identical either way.
 *   "graph_loop" GAC rounds (EAT/LD/REACH and SP/FP/LDS) as one CUDA graph with a
 *                conditional WHILE node (round number and stop test on the device):
 *                1 (default) = for graphs of >= 2^23 edges, 2 = always, 0 = never (host-
 *                driven rounds checked every "round_group" rounds); query lanes need it.
 *                Under a kernel profiler (ncu, compute-sanitizer) the rounds are host-driven
 *   "lanes"      1..4 (default 4): EAT/LD/REACH calls with several sub-batches and device
 *                outputs keep up to this many sub-batches in flight, one scratch set and
 *                stream each (as many sets as fit in device memory); 1 = one at a time */
TG_API tg_status tg_set_option(tg_graph *g, const char *key, int64_t value);

/* Total kernels this library has launched in this process (all handles). */
TG_API uint64_t tg_kernel_launch_count(void);

/* Device memory released by destroyed graphs is cached per device and reused by
 * later graphs / queries (no cudaMalloc / cudaFree per create-build-query cycle).
 * This returns every cached block to the CUDA driver. */
TG_API void tg_release_cached_memory(void);

/* Per-kernel timing for measurement: on = 1 brackets every launch with a CUDA
 * event pair recorded on the launching stream; on = 2 only the relaxation kernels
 * of the EAT family (activation, chunked ranges, chain walks: the roofline kernels),
 * which keeps the recording overhead out of the rest of the step; 0 = off.  tg_profile_report
 * synchronises on the recorded events and folds them into a per-kernel table;
 * with buf != NULL it writes the table as a JSON object
 * {"kernel_name": [launches, total_ms], ...} (NUL-terminated, truncated to
 * buf_len) and clears it; with buf == NULL it only returns the size.  Returns
 * the length needed (incl. NUL). */
TG_API void tg_profile_enable(int on);
TG_API int tg_profile_report(char *buf, uint64_t buf_len);

#ifdef __cplusplus
}
#endif
#endif /* TG_H */

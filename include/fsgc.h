/*
 * fsgc.h -- C ABI of the B200-native Fringe-SGC hot path.
 *
 * Method: Bradley, Alabandi, Burtscher, "Fringe-SGC: Counting Subgraphs with
 * Fringe Vertices", SC'25 (PAPER.md; citations are section / equation /
 * listing numbers because the extracted text is a single line).
 *
 * Three calls make up the path (north_star):
 *   fsgc_load_graph      edge list -> deduplicated, symmetrised, degree-ordered
 *                        CSR resident in device memory           (Sec. 2, 3.6)
 *   fsgc_compile_pattern core/fringe decomposition, fringe grouping by anchor
 *                        set, matching order, symmetry breaking,
 *                        automorphism count               (Def. 3.1-3.3, 3.4)
 *   fsgc_count           core matching + Venn diagram + fringe counting
 *                        function -> exact unsigned 128-bit counts
 *                                                     (Sec. 3.3-3.6, Listing 5)
 * Everything below is plain C: pointers and sizes, no C++ or torch types.
 *
 * Conventions
 *   - Every function returning int returns FSGC_OK (0) or an FSGC_ERR_* code;
 *     on error a human-readable message is available from fsgc_last_error()
 *     (thread-local) and output arguments are left unspecified.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *     stream).  Calls are stream-ordered; functions that return host values
 *     synchronise the stream before returning.
 *   - Vertex ids are 0-based.  Graph ids must be < num_vertices < 2^31.
 *   - Handles are owned by the caller and released with the matching
 *     fsgc_free_* call.  Handles may be shared read-only between threads, but
 *     concurrent fsgc_count calls on one graph must use different streams.
 *   - There is no CPU fallback: without a CUDA device every call that touches
 *     the device fails with FSGC_ERR_CUDA.  fsgc_compile_pattern and the
 *     pattern queries are host-only and work without a GPU.
 */
#ifndef FSGC_H
#define FSGC_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define FSGC_OK 0
#define FSGC_ERR_INVALID 1   /* bad argument (null pointer, id out of range, ...) */
#define FSGC_ERR_CUDA 2      /* CUDA runtime / driver error, or no device        */
#define FSGC_ERR_OOM 3       /* device allocation failed                         */
#define FSGC_ERR_PATTERN 4   /* pattern disconnected, invalid core, or beyond the
                                compiled limits (FSGC_MAX_*)                      */
#define FSGC_ERR_INTERNAL 5  /* an internal consistency check failed (bug)        */

#define FSGC_MAX_PATTERN_VERTICES 64  /* pattern vertex sets are 64-bit masks   */
#define FSGC_MAX_CORE 8               /* core vertices p                         */
#define FSGC_MAX_VENN_BITS 6          /* anchor vertices q per count pass        */
#define FSGC_MAX_BATCH 16             /* patterns per fsgc_count call            */

typedef struct fsgc_graph fsgc_graph;
typedef struct fsgc_pattern fsgc_pattern;

/* unsigned 128-bit integer, value = hi * 2^64 + lo */
typedef struct { uint64_t lo, hi; } fsgc_u128;

/* ------------------------------------------------------------------ graph */

/*
 * fsgc_load_graph -- build the device-resident CSR of a simple undirected
 * graph from an edge list (north_star "edge list -> deduplicated,
 * symmetrised, degree-ordered CSR"; Sec. 2 undirected graphs,
 * Sec. 3.6 degree-ordered matching / symmetry breaking by vertex id).
 *
 *   edges           num_input_edges pairs (a_i, b_i), row-major [E][2], of
 *                   int32 (index_bytes = 4) or int64 (index_bytes = 8).
 *                   Host memory if edges_on_device == 0 (copied with
 *                   cudaMemcpyAsync; pinned memory makes it asynchronous),
 *                   device memory otherwise.  Not retained after return.
 *   num_vertices    n; every id must be in [0, n).  Isolated vertices are
 *                   kept (they count for the 1-vertex pattern).
 *   Result          self loops dropped, duplicates and reversed duplicates
 *                   merged, each undirected edge stored in both directions.
 *                   Vertex ids are RELABELED: new id = rank of the vertex in
 *                   (degree ascending, original id ascending) order;
 *                   adjacency lists sorted ascending by new id.
 * Limits: n < 2^31 and, after deduplication, m < 2^31 undirected edges
 * (edge ids and CSR positions of the counting kernels are 32-bit: 2m must
 * fit an unsigned 32-bit index).  RMAT scale 26 (m = 1.05e9) fits.
 * Errors: FSGC_ERR_INVALID for null pointers, bad index_bytes, n <= 0 or
 * n >= 2^31, m >= 2^31 after deduplication, or an id outside [0, n)
 * (detected on the device); FSGC_ERR_OOM; FSGC_ERR_CUDA.  Synchronises
 * `stream`.
 */
int fsgc_load_graph(const void* edges, int64_t num_input_edges, int index_bytes,
                    int64_t num_vertices, int edges_on_device, void* stream,
                    fsgc_graph** out);

typedef struct {
    int64_t num_vertices;      /* n                                          */
    int64_t num_edges;         /* m, undirected edges after deduplication    */
    int64_t max_degree;
    /* device pointers, owned by the graph (valid until fsgc_free_graph)    */
    const int64_t* offsets;    /* [n+1] CSR row offsets                       */
    const int32_t* adj;        /* [2m]  neighbours, ascending per row         */
    const int32_t* row;        /* [2m]  row (source) of each CSR entry        */
    const int32_t* osrc;       /* [m]   oriented edges u<v, sorted (u, v) ... */
    const int32_t* odst;       /* [m]   ... as two arrays                     */
    const int32_t* order;      /* [n]   new id -> original id                 */
} fsgc_graph_info;

int fsgc_graph_get_info(const fsgc_graph* g, fsgc_graph_info* out);

/* Copy the CSR to host buffers of the sizes in fsgc_graph_info (any pointer
 * may be NULL to skip that array).  Synchronous. */
int fsgc_graph_download(const fsgc_graph* g, int64_t* offsets, int32_t* adj,
                        int32_t* order);

void fsgc_free_graph(fsgc_graph* g);

/* ---------------------------------------------------------------- pattern */

/*
 * fsgc_compile_pattern -- analyse a connected query pattern (host only).
 *
 *   num_vertices    P, 1 <= P <= FSGC_MAX_PATTERN_VERTICES
 *   edges           num_edges pairs (a, b), int32, row-major; loops and
 *                   duplicates are rejected
 *   core            NULL / core_size == 0: derive the core with the Sec. 3.4
 *                   heuristic (degree-1 vertices become tail fringes, then
 *                   degree-2 wedge fringes, ...; a disconnected core is
 *                   repaired by adding the shortest connecting path).
 *                   Otherwise the given core_size pattern vertices are the
 *                   core; they must induce a connected subgraph and every
 *                   other vertex may be adjacent only to core vertices
 *                   (Def. 3.1).
 * The handle records the core (<= FSGC_MAX_CORE vertices), its matching
 * order (Sec. 3.6: most constrained -- highest pattern degree -- first,
 * keeping connectivity), the fringe types (Def. 3.3: distinct anchor sets
 * and how many fringes share each), |Aut(P)| and prod k_t!.
 * Errors: FSGC_ERR_INVALID (null pointers, bad sizes), FSGC_ERR_PATTERN
 * (disconnected pattern, invalid core, limits exceeded).
 */
int fsgc_compile_pattern(int num_vertices, const int32_t* edges, int num_edges,
                         const int32_t* core, int core_size, fsgc_pattern** out);

typedef struct {
    int num_vertices;
    int num_edges;
    int core_size;                 /* p                                       */
    int32_t core_order[FSGC_MAX_CORE];   /* matching order, pattern ids      */
    int num_types;                 /* s, distinct anchor sets                 */
    uint64_t type_anchor[FSGC_MAX_PATTERN_VERTICES]; /* anchor set (bitmask of
                                      pattern vertex ids) of type t           */
    int32_t type_count[FSGC_MAX_PATTERN_VERTICES];   /* k_t                   */
    uint64_t core_mask;            /* bitmask of core pattern vertices        */
    uint64_t aut;                  /* |Aut(P)|                                */
    uint64_t aut_core;             /* |Aut(C)| of the unlabeled core          */
    uint64_t aut_core_labeled;     /* automorphisms of the core that map the
                                      fringe types onto types of equal k     */
    uint64_t fringe_factorial;     /* prod_t k_t!                             */
} fsgc_pattern_info;

int fsgc_pattern_get_info(const fsgc_pattern* p, fsgc_pattern_info* out);
void fsgc_free_pattern(fsgc_pattern* p);

/* ------------------------------------------------------------------ count */

typedef struct {
    fsgc_u128 count;        /* number of edge-induced embeddings of the pattern
                               (valid iff overflow == 0)                      */
    fsgc_u128 raw;          /* sum of fc over the enumerated core instances
                               and fringe programs, before scaling            */
    uint64_t divisor;       /* count = raw / divisor (exact)                  */
    uint64_t core_matches;  /* core instances enumerated by this call         */
    int32_t overflow;       /* 1 if an intermediate or the result exceeded
                               2^128 - 1: count is then not valid             */
    int32_t root_pattern_vertex; /* pattern vertex matched at the root (c0)  */
    float kernel_ms;        /* device time of this pattern's counting kernel
                               (CUDA events around the launch on `stream`)    */
    float aux_ms;           /* device time of the auxiliary per-edge support
                               pass (edge cores), 0 otherwise                 */
    int32_t kernel_launches;/* kernels launched for this pattern's pass       */
    int32_t pass_index;     /* patterns with equal pass_index shared one pass */
    int32_t pass_kind;      /* 0 vertex core, 1 edge core (support + fc),
                               2 general core, 3 triangle core (support + tri) */
} fsgc_result;

typedef struct {
    int64_t root_begin;     /* root item range [root_begin, root_end) ...     */
    int64_t root_end;       /* ... (root_end < 0: all items)                  */
    int32_t shard_index;    /* this process's shard (0 if unsharded)          */
    int32_t shard_count;    /* shards; root chunks are dealt round-robin      */
    int32_t no_symmetry_breaking; /* 1: enumerate every injective core map, one
                               fringe program (used for per-root checks)      */
    int32_t flags;          /* FSGC_FLAG_* bits                               */
} fsgc_count_opts;

/* disable the degree filter (Sec. 3.6 "degree filtering"): every core
 * instance is visited, so fsgc_result.core_matches is the number of core
 * instances in the graph (within the root range) */
#define FSGC_FLAG_NO_DEGREE_FILTER 1
/* multi-GPU (north_star "root-edge ranges are sharded"): with shard_count > 1
 * the per-edge support pass c(e) = |N(u) & N(v)| (the oriented triangle
 * listing that edge, triangle and general cores read) is sharded too: shard s
 * lists the triangles of the support-order chunks s, s + shard_count, ...
 * into a partial array, and the caller SUMS the shards' partial arrays (one
 * all-reduce of int32[m], fsgc_plan_support_region) between the two stages of
 * fsgc_plan_enqueue_stage.  Without the flag every shard computes the whole
 * support array itself (no exchange).  fsgc_count rejects the flag. */
#define FSGC_FLAG_SHARD_SUPPORT 2

/*
 * fsgc_count -- count npats patterns on graph g in ONE pass over the core
 * matches when their cores are isomorphic (the Venn diagram of a core match
 * is computed once and every pattern's fringe programs are evaluated on it);
 * patterns with different cores are grouped and counted pass by pass.
 *
 *   pats / npats    1 <= npats <= FSGC_MAX_BATCH compiled patterns
 *   results         host array [npats]
 *   opts            NULL = whole graph, symmetry breaking on, one shard.
 *                   Root items are the units of work (Sec. 3.6 "each thread
 *                   starts from a distinct graph vertex"; here: root edges,
 *                   or vertices for 1-vertex cores); see fsgc_num_roots.
 *                   With shard_count > 1 the caller combines the `raw`
 *                   values of all shards (sum, e.g. an NCCL all-reduce) and
 *                   calls fsgc_finalize.
 * Method: Sec. 3 -- each core instance (one per automorphism orbit of the
 * core, symmetry breaking per Sec. 3.1) gets the sizes of the 2^q - 1
 * disjoint regions of its anchors' external neighbour sets (Sec. 3.3/3.4),
 * and fc (Listing 5) counts the fringe completions; count = raw * |Aut_C'|
 * * prod k_t! / |Aut(P)| (Sec. 3.1 "divide the final count by the number of
 * automorphisms").  Exact 128-bit arithmetic with overflow detection.
 * Errors: FSGC_ERR_INVALID, FSGC_ERR_PATTERN (q > FSGC_MAX_VENN_BITS),
 * FSGC_ERR_CUDA, FSGC_ERR_OOM.  Synchronises `stream`.
 */
int fsgc_count(const fsgc_graph* g, const fsgc_pattern* const* pats, int npats,
               const fsgc_count_opts* opts, fsgc_result* results, void* stream);

/* Number of root items of the pass that counts pattern p (with the given
 * symmetry mode): m (oriented root edges), 2m (directed root edges) or n
 * (vertices, 1-vertex cores); 0 for the 1- and 2-vertex patterns. */
int fsgc_num_roots(const fsgc_graph* g, const fsgc_pattern* p,
                   int no_symmetry_breaking, int64_t* out);

/* Turn a (summed) raw value into the final count: count = raw / divisor,
 * where divisor is taken from a result of the same pattern and mode. */
int fsgc_finalize(fsgc_u128 raw, uint64_t divisor, int32_t overflow,
                  fsgc_u128* count, int32_t* count_overflow);

/* ------------------------------------------------------------- plans */
/*
 * Reusable, CUDA-graph-capturable execution of fsgc_count.
 *
 *   fsgc_plan_create      host: group the patterns into passes, build the
 *                         fringe programs, size the grids and the workspace
 *                         (initialises the device binomial table once per
 *                         device, synchronously).  The plan keeps pointers to
 *                         `g` and must not outlive it.
 *   fsgc_plan_workspace_bytes  device workspace size (*ws) and raw result
 *                         block size (*raw) the plan needs
 *   fsgc_plan_enqueue     stream-ordered: zero the workspace header, run
 *                         every pass's kernels, copy the raw 128-bit sums and
 *                         flags to `raw_out` (device or pinned host memory,
 *                         *raw bytes).  No allocation and no host
 *                         synchronisation, so it can be captured in a CUDA
 *                         graph.  One plan must not be enqueued concurrently
 *                         on two streams with the same workspace.
 *   fsgc_plan_decode      after the stream completed: raw block -> results
 *                         (as fsgc_count returns them; kernel_ms / aux_ms are
 *                         best effort, -1 when unavailable)
 */
typedef struct fsgc_plan fsgc_plan;

int fsgc_plan_create(const fsgc_graph* g, const fsgc_pattern* const* pats, int npats,
                     const fsgc_count_opts* opts, fsgc_plan** out);
int fsgc_plan_workspace_bytes(const fsgc_plan* plan, size_t* ws, size_t* raw);
int fsgc_plan_enqueue(const fsgc_plan* plan, void* workspace, void* raw_out, void* stream);

/*
 * Staged enqueue (same rules as fsgc_plan_enqueue; stages is a bit mask):
 *   FSGC_STAGE_SUPPORT  zero the support array and run the support pass
 *                       (this shard's part with FSGC_FLAG_SHARD_SUPPORT)
 *   FSGC_STAGE_COUNT    every pass's counting kernel (reads the support
 *                       array as it is in the workspace) + the raw copy
 * fsgc_plan_enqueue == both stages; it fails with FSGC_ERR_INVALID for a
 * plan whose support pass is sharded.
 * fsgc_plan_support_region: the support array is int32[*count] at byte
 * *offset of the workspace (*count = 0: no pass of the plan reads it).  It
 * is indexed by oriented edge (u < v) in (u, v) order.
 */
#define FSGC_STAGE_SUPPORT 1
#define FSGC_STAGE_COUNT 2
#define FSGC_STAGE_ALL 3
int fsgc_plan_enqueue_stage(const fsgc_plan* plan, void* workspace, void* raw_out, int stages,
                            void* stream);
int fsgc_plan_support_region(const fsgc_plan* plan, size_t* offset, int64_t* count);
int fsgc_plan_decode(const fsgc_plan* plan, const void* raw, fsgc_result* results);
void fsgc_plan_free(fsgc_plan* plan);

/* thread-local message for the last failing call ("" if none) */
const char* fsgc_last_error(void);

/* library version string */
const char* fsgc_version(void);

#ifdef __cplusplus
}
#endif
#endif /* FSGC_H */

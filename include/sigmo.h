/*
 * sigmo.h -- C ABI of the B200-native SIGMo hot path (libsigmo.so).
 *
 * SIGMo: batched molecular subgraph isomorphism (De Caro et al., SC '25;
 * /root/reference/PAPER.md, cited as P:<line>).  The library computes, for
 * every (query graph q, data graph g) pair of a batch, the number of
 * label- and bond-preserving injective maps V_q -> V_g (Find All) or whether
 * one exists (Find First):
 *   problem  : Def. 2.1, NLSM, bond labels checked
 *              (P:724-726); non-induced reading R1, mappings counted R2;
 *   modes    : Find All / Find First;
 *   pipeline : CSR-GO load (section 4.1) -> multi-level signature
 *              filter (Alg. 1; section 4.2-4.4) ->
 *              GMCR mapping (section 4.5) -> DFS join
 *              (section 4.6).
 * Readings of the paper (R1-R21) are listed in DESIGN.md.
 *
 * Conventions (all calls):
 *   * Every call returns sigmo_status; 0 = SIGMO_OK.  On error the context
 *     keeps a message readable with sigmo_last_error(ctx).  No C++ exception
 *     crosses the ABI; bad input never aborts.
 *   * Host pointers passed in are read during the call only, never retained.
 *     Output buffers are caller-allocated; sizes are obtained first.
 *   * All device work is enqueued on the context's CUDA stream.  Getters that
 *     return host data synchronize that stream before returning.
 *   * State machine: load_batch -> filter -> join -> get_*.  Out-of-order
 *     calls return SIGMO_ERR_STATE.  A new load_batch invalidates results;
 *     filter may be re-run with other levels/flags, join with other modes.
 *   * A context is bound to one device and one stream; it is not thread-safe.
 */
#ifndef SIGMO_H_
#define SIGMO_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define SIGMO_API __attribute__((visibility("default")))
#else
#define SIGMO_API
#endif

typedef enum {
  SIGMO_OK = 0,
  SIGMO_ERR_INVALID_ARG = -1,   /* NULL pointer, bad enum, levels out of range, buffer too small */
  SIGMO_ERR_INVALID_GRAPH = -2, /* malformed CSR-GO (see sigmo_load_batch) */
  SIGMO_ERR_LIMIT = -3,         /* a documented size limit is exceeded */
  SIGMO_ERR_STATE = -4,         /* call out of order (e.g. join before filter) */
  SIGMO_ERR_OOM = -5,           /* device allocation failed */
  SIGMO_ERR_CUDA = -6           /* CUDA runtime error (message has the CUDA text) */
} sigmo_status;

/* Join modes. */
typedef enum { SIGMO_FIND_ALL = 0, SIGMO_FIND_FIRST = 1 } sigmo_mode;

/* sigmo_filter flags.  NEIGHBOR_SUPPORT: after the signature levels, remove
 * v_d from C(v_q) while some query edge (v_q,u_q,b) has no data edge
 * (v_d,u_d,b) with u_d in C(u_q); iterate to the unique greatest fixed point
 * (BASELINE.json north_star; not in the paper -- DESIGN.md R9). */
enum { SIGMO_FILTER_NEIGHBOR_SUPPORT = 1u << 0 };

/* Limits (SIGMO_ERR_LIMIT). */
enum {
  SIGMO_MAX_QUERY_NODES = 32,  /* paper: queries <= 30 nodes */
  SIGMO_MAX_DATA_NODES = 256,  /* per data graph; fast path <= 64 */
  SIGMO_MAX_LEVELS = 16,
  SIGMO_MAX_BOND_CLASSES = 8   /* distinct bond labels among query edges */
};

typedef struct sigmo_ctx sigmo_ctx; /* opaque */

/* A CSR-GO batch (section 4.1; Fig. 3): all graphs of
 * the batch form one disconnected graph.  Host pointers.
 *   graph_offsets[num_graphs+1] : node id of each graph's first node,
 *                                 graph_offsets[0]=0, non-decreasing,
 *                                 graph_offsets[num_graphs]=num_nodes
 *   row_offsets[num_nodes+1]    : CSR row offsets, row_offsets[0]=0
 *   col_indices[row_offsets[num_nodes]] : GLOBAL node ids, both directions
 *                                 of every undirected edge
 *   node_labels[num_nodes]      : atom label (atomic number by convention)
 *   edge_labels[row_offsets[num_nodes]] : bond label per adjacency entry
 *                                 (1 single, 2 double, 3 triple, 4 aromatic
 *                                 by convention; any u8 allowed, equality only) */
typedef struct {
  int64_t num_graphs, num_nodes;
  const int64_t *graph_offsets;
  const int64_t *row_offsets;
  const int32_t *col_indices;
  const uint8_t *node_labels;
  const uint8_t *edge_labels;
} sigmo_graph_batch;

/* Optional device allocator (e.g. the PyTorch caching allocator).  alloc must
 * return device memory usable on `stream`, or NULL on failure. */
typedef struct {
  void *(*alloc)(size_t bytes, void *stream, void *user);
  void (*free)(void *ptr, void *stream, void *user);
  void *user;
} sigmo_allocator;

/* Per-stage device times (ms), averaged over the filter/join calls made with
 * timing enabled since the previous sigmo_get_timings (which resets them).
 * CUDA events are recorded on the ctx stream around each kernel; recording
 * never synchronizes, sigmo_get_timings does.  0 for stages not run. */
typedef struct {
  float query_prep_ms;  /* query signatures + plane/row programs (built once per levels) */
  float filter_ms;      /* fused signature + dominance + bitmap + GMCR-test kernel */
  float support_ms;     /* neighbour-support fixed point (0 if flag off) */
  float mapping_ms;     /* GMCR scan + join chunking */
  float join_ms;        /* DFS join kernel (incl. per-query totals) */
  int64_t filter_launches, join_launches;  /* kernels launched by the last filter / join call */
  int64_t h2d_bytes;    /* bytes uploaded by the last sigmo_load_batch (one pinned H2D copy) */
  int64_t filter_calls, join_calls;        /* calls averaged */
  int64_t dfs_steps;    /* DFS iterator steps (search-tree nodes) of the last join (counted only
                           with sigmo_set_timing bit 1; else 0 on the lane path) */
  int64_t dfs_iters, dfs_tail_iters, dfs_max_stack;  /* warp iterations, of which after the last pair claim; max stack */
  int64_t filter_jit;   /* 1 if the last lane-path filter ran the kernel specialised for the query program (NVRTC) */
  double jit_compile_ms; /* wall time of the last specialisation compile (0 if served from the process cache) */
} sigmo_timings;

/* Create a context on `device` (CUDA ordinal) enqueuing on `cuda_stream`
 * (a cudaStream_t; NULL = the legacy default stream).  alloc NULL ->
 * cudaMallocAsync/cudaFreeAsync on the stream.  *out receives the context. */
SIGMO_API sigmo_status sigmo_create(int device, void *cuda_stream, const sigmo_allocator *alloc, sigmo_ctx **out);

/* Validate, pack and upload one query batch and one data batch (step S1).
 * Rejected with SIGMO_ERR_INVALID_GRAPH: offsets not starting at 0 or
 * decreasing, num_nodes inconsistent, a column outside the owning graph,
 * self-loops, duplicate edges, asymmetric adjacency, an edge label that
 * differs between (u,v) and (v,u), an empty (0-node) query graph.
 * SIGMO_ERR_LIMIT: a query graph > 32 nodes, a data graph > 256 nodes,
 * > 2^31-1 nodes or adjacency entries, > 8 distinct query bond labels.
 * Disconnected graphs and single-node queries are accepted; an empty data
 * batch is accepted (all results empty).  Blocks until the inputs are
 * packed into pinned staging memory; the upload is asynchronous. */
SIGMO_API sigmo_status sigmo_load_batch(sigmo_ctx *ctx, const sigmo_graph_batch *queries, const sigmo_graph_batch *data);

/* Build the candidate bitmap C_L (Alg. 1) and the GMCR.
 * levels L in 1..16 (reading R6): L=1 -> labels only (InitializeCandidates,
 * Alg.1 l.29-37); L>=2 also applies signature dominance at radii 1..L-1
 * (GenerateSignatures l.11-18 cumulative per R4, RefineCandidates l.19-28 on
 * every field per R5, saturating fields per R7/R8).  flags: 0 or
 * SIGMO_FILTER_NEIGHBOR_SUPPORT.  With the flag, the lane path (graphs <= 64
 * atoms, queries <= 11 nodes) refines the candidate windows of every GMCR
 * pair to the fixed point (k_support_lane) and the join reads the refined
 * windows; the general path runs k_support over the dense bitmap.
 * Asynchronous, except that the first call for a given `levels` after
 * load_batch synchronizes once to size the query-side plane program, and
 * the lane-path neighbour-support pass synchronizes once to size its
 * per-pair window arrays. */
SIGMO_API sigmo_status sigmo_filter(sigmo_ctx *ctx, int levels, uint32_t flags);

/* Stack-based DFS join over the GMCR pairs (section 4.6).
 * FIND_ALL: per-pair u64 embedding counts; FIND_FIRST: per-pair 0/1.
 * Also accumulates per-query totals (sum over data graphs).  If
 * total_matches_out (host) is non-NULL, it receives the sum over all pairs
 * (synchronizes); otherwise the call is asynchronous. */
SIGMO_API sigmo_status sigmo_join(sigmo_ctx *ctx, sigmo_mode mode, uint64_t *total_matches_out);

/* Number of (query, data graph) pairs that survived the GMCR rule (after filter). */
SIGMO_API sigmo_status sigmo_num_pairs(sigmo_ctx *ctx, int64_t *n_pairs);

/* Sparse per-pair results after join, grouped by data graph ascending, then
 * query ascending.  cap = capacity of the three host arrays; *n receives the
 * number of pairs (SIGMO_ERR_INVALID_ARG if cap < n; n is still set).
 * result: count (FIND_ALL) or 0/1 (FIND_FIRST).  Any array may be NULL. */
SIGMO_API sigmo_status sigmo_get_pair_results(sigmo_ctx *ctx, int64_t cap, int64_t *n, int64_t *data_idx,
                                    int32_t *query_idx, uint64_t *result);

/* Dense results out[q*num_data_graphs + g] (host, NQ*ND u64); pairs pruned by
 * the GMCR are 0.  Intended for small batches and tests. */
SIGMO_API sigmo_status sigmo_get_dense_results(sigmo_ctx *ctx, uint64_t *out);

/* Per-query totals (sum over data graphs of the join results), NQ u64.
 * device_ptr = 0: `out` is host memory (synchronizes); 1: `out` is device
 * memory on this ctx's device (asynchronous copy on the ctx stream). */
SIGMO_API sigmo_status sigmo_get_query_totals(sigmo_ctx *ctx, uint64_t *out, int device_ptr);

/* Candidate bitmap view (reading R10): host out[VQ*ceil(VD/32)] u32,
 * row = global query node, bit j of word w = data node 32w+j (LSB-first). */
SIGMO_API sigmo_status sigmo_get_candidates(sigmo_ctx *ctx, uint32_t *out);

/* Packed masked-bitset signatures (section 4.2; field table R7,
 * saturation R8) at `radius` in 1..255 of every node: which = 0 queries, 1 data.
 * Host out[V] u64.  Requires load_batch only. */
SIGMO_API sigmo_status sigmo_get_signatures(sigmo_ctx *ctx, int which, int radius, uint64_t *out);

/* ---- Embedding enumeration ----
 * NLSM's literal output is the set of embeddings X and atom typing
 * needs every isomorphism, not a count.  sigmo_enumerate runs, on
 * the device, a Find All count pass of the join, a prefix sum of the per-pair
 * counts (each pair's first slot) and a write pass in which every leaf of the
 * DFS writes its mapping f.  flags SIGMO_ENUM_NODE_SETS also forms, per pair,
 * the distinct node sets f(V_q) (automorphic images collapse to one set) as
 * molecule-local 64-bit masks.  Requires sigmo_filter (any levels and flags)
 * on the lane path: every data
 * graph <= 64 atoms and every query <= 11 nodes; else SIGMO_ERR_LIMIT.  The
 * per-pair results of the last join are the Find All counts afterwards.
 * *num_embeddings (nullable) = the total.  Device memory: stride (8 bytes for
 * queries <= 8 nodes, else 16) per embedding, + 8 with node sets. */
enum { SIGMO_ENUM_NODE_SETS = 1u << 0 };
SIGMO_API sigmo_status sigmo_enumerate(sigmo_ctx *ctx, uint32_t flags, int64_t *num_embeddings);
/* Copy the embeddings of the last sigmo_enumerate to the host, pairs in the
 * order of sigmo_get_pair_results (data graph, then query).  Call with NULL
 * arrays to get *num_pairs, *num_embeddings and *stride.  Then
 * data_idx/query_idx[num_pairs], emb_offsets[num_pairs+1] (embeddings of pair
 * k are [emb_offsets[k], emb_offsets[k+1])), maps[num_embeddings * stride]:
 * byte i of an embedding = molecule-local index of the data node that query
 * node i maps to (0xff.. padding beyond the query's size is 0). */
SIGMO_API sigmo_status sigmo_get_embeddings(sigmo_ctx *ctx, int64_t pair_cap, int64_t *num_pairs, int64_t *data_idx,
                                            int32_t *query_idx, int64_t *emb_offsets, int64_t emb_cap, uint8_t *maps,
                                            int64_t *num_embeddings, int32_t *stride);
/* The distinct node sets (SIGMO_ENUM_NODE_SETS), same pair order: bit j of a
 * set = molecule-local data node j; sets of a pair ascending.  NULL arrays:
 * sizes only. */
SIGMO_API sigmo_status sigmo_get_node_sets(sigmo_ctx *ctx, int64_t pair_cap, int64_t *num_pairs, int64_t *set_offsets,
                                           int64_t set_cap, uint64_t *sets, int64_t *num_sets);

/* Read back the CSR-GO batch as the library packed it on the device
 * (section 4.1; Fig. 3): which = 0 queries, 1 data.
 * sizes: *num_graphs, *num_nodes, *num_adj (adjacency entries, both
 * directions).  Pass NULL arrays to query the sizes only; otherwise
 * caller-allocated host arrays graph_offsets[G+1], row_offsets[V+1],
 * col_indices[E2] (global node ids), node_labels[V], edge_labels[E2] are
 * filled from the device arrays (a test hook that pins the packer against
 * the paper's worked example).  Requires load_batch.  Synchronizes. */
SIGMO_API sigmo_status sigmo_get_packed_batch(sigmo_ctx *ctx, int which, int64_t *num_graphs, int64_t *num_nodes,
                                              int64_t *num_adj, int64_t *graph_offsets, int64_t *row_offsets,
                                              int32_t *col_indices, uint8_t *node_labels, uint8_t *edge_labels);

/* SIGMO_OK if the last sigmo_join completed within the kernels' internal
 * capacities, else SIGMO_ERR_LIMIT (the results are then incomplete).  The
 * device-pointer path of sigmo_get_query_totals does not synchronize, so
 * callers that only read totals on the device (multi-GPU all-reduce,
 * streaming) check this once per run.  Synchronizes. */
SIGMO_API sigmo_status sigmo_check_join(sigmo_ctx *ctx);

/* Induced-subgraph mode (the literal G_D[X] reading of
 * Def. 2.1; R21): an embedding must also map every
 * NON-adjacent query node pair to a non-adjacent data node pair (a data bond
 * of any label counts as adjacency).  enable = 0 (default, monomorphism,
 * reading R1) or 1.  Takes effect at the next sigmo_load_batch; both join
 * kernels (the per-lane k_join_lane and the general k_join) apply the
 * non-edge constraints; the filter is unchanged (induced embeddings are a
 * subset of the monomorphisms, so its candidate sets stay sound).  Never
 * fails for a valid ctx. */
SIGMO_API sigmo_status sigmo_set_induced(sigmo_ctx *ctx, int enable);
/* Wildcard atoms and bonds (the paper's stated next step,
 * P:2639-2645; R22): with enable = 1, a QUERY atom label 0 is the
 * SMARTS '*' (matches an atom of any label) and a query bond label 0 the
 * SMARTS '~' (matches a bond of any label); data labels stay literal.  Takes
 * effect at the next sigmo_load_batch.  The filter stays sound: a '*' atom's
 * candidates start from every atom and it adds to no signature field of the
 * other query atoms; '~' bonds use the all-bond adjacency in the join and in
 * the neighbour-support pass.  With '~' bonds at most 7 distinct concrete
 * query bond labels (SIGMO_ERR_LIMIT).  The query side of
 * sigmo_get_signatures leaves '*' atoms out of every field.  Never fails for a
 * valid ctx. */
SIGMO_API sigmo_status sigmo_set_wildcards(sigmo_ctx *ctx, int enable);
/* Per-stage CUDA-event timing and DFS step counting (default off), and their
 * read-out.  enable bit 0: CUDA events around the filter, mapping and join
 * stages; bit 1: the join counts its DFS steps (sigmo_timings.dfs_steps; the
 * lane join then runs its counting instantiation instead of the lean one, so
 * time it with bit 1 clear).  Other bits are ignored.  Never fails for a
 * valid ctx. */
SIGMO_API sigmo_status sigmo_set_timing(sigmo_ctx *ctx, int enable);
SIGMO_API sigmo_status sigmo_get_timings(sigmo_ctx *ctx, sigmo_timings *out);

/* Host-only structural validation of one batch (no device needed): the
 * checks of sigmo_load_batch for a query (is_query=1) or data batch.
 * msg (nullable) receives a NUL-terminated reason. */
SIGMO_API sigmo_status sigmo_validate_batch(const sigmo_graph_batch *batch, int is_query, char *msg, size_t msg_len);

/* Message of the last error on this context ("" if none).  Valid until the
 * next call on the context. */
SIGMO_API const char *sigmo_last_error(const sigmo_ctx *ctx);

/* Library version string, e.g. "sigmo-b200 0.1". */
SIGMO_API const char *sigmo_version(void);

/* Release all device and host resources of the context (synchronizes). */
SIGMO_API sigmo_status sigmo_destroy(sigmo_ctx *ctx);

#ifdef __cplusplus
}
#endif
#endif /* SIGMO_H_ */

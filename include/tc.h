/*
 * tc.h — C-ABI of the B200 intersection-based triangle counting (ITC) library.
 *
 * The operation (PAPER.md = Li et al., "A Comparative Study of
 * Intersection-Based Triangle Counting Algorithms on GPUs", IPDPS-W 2024):
 *
 *   T(G) = |{ {x,y,z} : {x,y}, {y,z}, {x,z} in E }|
 *
 * for the simple undirected graph G obtained from a raw edge list by
 * ignoring direction, dropping self-loops and merging duplicates (P:287:
 * cleaning "do[es] not alter the number of triangles").  The library
 * reaches T exactly by the edge-iterator intersection of P:78 (Fig. 1(b))
 * over a degree-oriented DAG: every triangle u<v<w (in the
 * orientation order) is found once, at oriented edge (u,v), as the witness
 * w in N+(u) ∩ N+(v).  Counts are exact integers; there is no rounding.
 *
 * Pipeline:
 *   tc_build_csr  : a1 validate + canonicalise + drop self-loops,
 *                   a2 radix sort + unique, a3 degree, a4 rank by
 *                   (degree, id) + relabel + drop isolated vertices,
 *                   a5 orient + per-row sort -> CSR, a6 dispatch plan.
 *   tc_count*     : a7/a8 grouped counting kernels, a9 u64 reduction.
 *
 * Conventions (all entry points):
 *   - extern "C", return tc_status, never throw, never abort.
 *   - Device pointers are CUDA device memory of the current device; host
 *     pointers are ordinary (pageable or pinned) host memory.
 *   - `stream` is a cudaStream_t passed as void* (0 = legacy default
 *     stream).  Work is stream ordered; only functions that write a host
 *     output (h_*) synchronise the stream.
 *   - Vertex ids are int32 (0 <= id < 2^31-1); edge counts and offsets are
 *     int64; triangle counts are uint64 (they exceed 2^32 at config C3).
 *   - On any non-OK status, tc_last_error() returns a thread-local message.
 *   - A tc_graph is immutable after tc_build_csr / tc_replan returns, so
 *     concurrent counts on one graph from different streams are allowed.
 */
#ifndef TC_H
#define TC_H
#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define TC_API __attribute__((visibility("default")))
#else
#define TC_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  TC_OK = 0,
  TC_ERR_INVALID_ARGUMENT = 1, /* null pointer, id out of range, bad range   */
  TC_ERR_OUT_OF_MEMORY = 2,    /* the allocator returned NULL                */
  TC_ERR_CUDA = 3,             /* a CUDA runtime error (text in tc_last_error) */
  TC_ERR_UNSUPPORTED = 4       /* a size the library does not handle          */
} tc_status;

typedef struct tc_graph tc_graph; /* opaque: owns the device CSR and plan */

/* Build flags. */
#define TC_KEEP_ISOLATED 0x1u /* keep degree-0 vertices as empty rows (n' = n) */

/*
 * Device allocator hook.  alloc returns NULL on failure (-> TC_ERR_OUT_OF_MEMORY);
 * free receives exactly the pointer/size/stream of a prior alloc.  The default
 * (tc_set_allocator(NULL, NULL, NULL)) is cudaMallocAsync / cudaFreeAsync on
 * the calling stream.  Process-wide; set it before building graphs.
 */
typedef void* (*tc_alloc_fn)(size_t bytes, void* stream, void* ctx);
typedef void (*tc_free_fn)(void* ptr, size_t bytes, void* stream, void* ctx);
TC_API tc_status tc_set_allocator(tc_alloc_fn alloc, tc_free_fn free_fn, void* ctx);

/*
 * Plan options (performance parameters that never
 * change the count; the property tests vary them).  0 in a field = default.
 */
typedef struct {
  int32_t chunk_cost;   /* cost units per work chunk (default 16384)               */
  int32_t seg_cost;     /* fixed cost per live oriented edge (default 4)          */
  int32_t huge_degree;  /* d+(v) above which N+(v) is probed in global memory by
                           binary search instead of an SMEM hash (default 8192)    */
  int32_t block_threads;/* threads per CTA of the long-class count kernel,
                           64..1024; 1/4 of the warps (TC_PROD_DIV) build tables in
                           two groups, the rest probe (default 1024)                                          */
  int32_t table_factor; /* hash slots = table_factor * d+(v) (rounded up to a
                           multiple of 4), 2..16 (default 6, i.e. load <= 1/6)     */
  int32_t long_min;     /* trimmed suffixes with >= long_min keys go to the
                           warp-per-edge tile class, shorter ones to the flattened
                           class (default 32; values below 32 act as 32, since a
                           tile holds 32 keys of its own edge; 2^30 = all short).
                           Edges whose head gets a hash table with d+(v) <= 128
                           are flattened whatever their length (env
                           TC_LONG_HASH_DMAX; 0 = pure length split)         */
  int32_t probe_mode;   /* 0 = two-choice (cuckoo) tables with linear-probing
                           fallback per chunk, 1 = linear probing only (default 0) */
  int32_t bitmap_factor; /* a head v whose window [min N+(v), max N+(v)] needs at most
                           bitmap_factor * d+(v) 32-bit words gets a bitmap table
                           (one probe per key) instead of a hash table (two);
                           default 16, -1 = never                                */
} tc_options;

/*
 * a1..a6.  Build the oriented CSR and dispatch plan from a raw edge list.
 *   d_src, d_dst : device int32[num_edges]; pair i is the undirected edge
 *                  {d_src[i], d_dst[i]}.  Caller-owned, never modified.
 *                  Duplicates, reversed pairs and self-loops are allowed
 *                  (cleaned).
 *   num_edges    : >= 0; 0 gives a valid empty graph (T = 0).
 *   num_vertices : ids must lie in [0, num_vertices); -1 = max id + 1.
 *   flags        : TC_KEEP_ISOLATED or 0.
 *   opts         : NULL for defaults.
 *   out          : receives the new graph; NULL on any error (nothing leaks).
 * Errors: TC_ERR_INVALID_ARGUMENT for null pointers, num_edges < 0,
 * num_vertices > 2^31-1, or any id < 0 or >= num_vertices.
 * Synchronises `stream` (the unique-edge count must reach the host).
 */
TC_API tc_status tc_build_csr(const int32_t* d_src, const int32_t* d_dst, int64_t num_edges,
                       int64_t num_vertices, uint32_t flags, const tc_options* opts,
                       void* stream, tc_graph** out);

/* Same, from HOST int32 arrays: the library copies them to the device on
 * `stream` first (the end-to-end entry point bench.py's e2e leg times). */
TC_API tc_status tc_build_csr_host(const int32_t* h_src, const int32_t* h_dst, int64_t num_edges,
                            int64_t num_vertices, uint32_t flags, const tc_options* opts,
                            void* stream, tc_graph** out);

/* Rebuild only the dispatch plan (a6) with new options. */
TC_API tc_status tc_replan(tc_graph* g, const tc_options* opts, void* stream);

typedef struct {
  int64_t n_input;          /* num_vertices as given / inferred                 */
  int64_t n;                /* n': rows of the CSR (non-isolated vertices)      */
  int64_t m;                /* unique undirected edges = oriented edges |E+|    */
  int64_t max_out_degree;   /* max d+(u)                                        */
  int64_t m_live;           /* oriented edges with non-empty work (plan units)  */
  int64_t n_groups;         /* distinct middle vertices v with live edges       */
  int64_t n_chunks;         /* work chunks of the count kernel                  */
  int64_t keys_total;       /* sum of suffix lengths over live edges (probes)   */
  uint64_t b_itc;           /* algorithmic bytes B_ITC         */
  int64_t smem_bytes;       /* dynamic SMEM per CTA of the count kernel          */
  int32_t count_grid;       /* CTAs the count kernel launches                    */
  int32_t count_block;      /* threads per CTA                                   */
  /* Borrowed device pointers, valid until tc_free: */
  const int64_t* row_ptr;   /* int64[n+1], row offsets of the oriented CSR       */
  const int32_t* col;       /* int32[m], each row strictly ascending, col > row  */
  const int32_t* perm;      /* int32[n], new id -> original id                   */
  /* Build phase times (ms, CUDA events on the build stream): */
  float ms_canon, ms_sort_unique, ms_degree_rank, ms_orient_csr, ms_plan, ms_total;
  int64_t n_long_chunks;    /* chunks [0, n_long_chunks) are long class (k_count),
                               the rest short class (k_count_flat): a count launches
                               one kernel per non-empty class                       */
  /* The method's own bytes: what one full count reads from
   * memory as designed, every element once per use — the 4-B key of every
   * trimmed suffix position (4 * keys_total), the plan entries of every live
   * edge, and per (chunk, group) pair the head's row N+(v) (4 * d+(v)) and its
   * group entries, plus the chunk bounds.  The count step's roofline bytes. */
  uint64_t method_bytes;
  int64_t table_words;      /* sum over (chunk, group) pairs of d+(v)             */
  int64_t group_visits;     /* number of (chunk, group) pairs                     */
  int64_t m_live_long;      /* live edges [0, m_live_long) are long class         */
  uint64_t method_bytes_long; /* the long class's part of method_bytes            */
  int64_t keys_long;        /* trimmed keys of the long class                      */
} tc_graph_info_t;

TC_API tc_status tc_graph_info(const tc_graph* g, tc_graph_info_t* out);

/* a7..a9.  T of the whole graph.  h_count: host uint64.  Synchronises. */
TC_API tc_status tc_count(const tc_graph* g, void* stream, uint64_t* h_count);

/* Stream-ordered variant: writes T into device uint64 *d_count (no sync). */
TC_API tc_status tc_count_async(const tc_graph* g, void* stream, uint64_t* d_count);

/*
 * Partial count over the live oriented edges [e_begin, e_end) of the plan
 * order (0 <= e_begin <= e_end <= m_live): writes sum_{e in range} |N+(u_e) ∩
 * N+(v_e)| into device uint64 *d_partial (overwritten, not accumulated).
 * Any cut of [0, m_live) into ranges gives partials summing to T (P:78:
 * the per-edge intersections are independent).  No sync.
 */
TC_API tc_status tc_count_range(const tc_graph* g, int64_t e_begin, int64_t e_end, void* stream,
                         uint64_t* d_partial);

/*
 * Per-edge triangle support (the k-truss and
 * clustering-coefficient inputs P:39 names): d_support (device uint32[m],
 * caller-owned, overwritten) receives, for every CSR edge position p in
 * [0, m), the number of triangles of G that contain the undirected edge
 * {row(p), col[p]} (= |N(a) ∩ N(b)| over full neighbourhoods).  Every
 * triangle u<v<w found at oriented edge (u,v) with witness w
 * adds 1 to (u,v), (u,w) and (v,w), so sum(d_support) = 3T.  Use
 * tc_edge_list to map positions to original vertex ids.  No sync; needs
 * 8 B x m_live of stream-ordered scratch.  Errors: NULL graph or output ->
 * TC_ERR_INVALID_ARGUMENT; tables that would exceed SMEM in support layout
 * -> TC_ERR_UNSUPPORTED (rebuild with a lower huge_degree).
 */
TC_API tc_status tc_support(const tc_graph* g, void* stream, uint32_t* d_support);

/*
 * Original vertex ids of every CSR edge: d_u[p] = perm[row(p)], d_v[p] =
 * perm[col[p]] for p in [0, m) (device int32[m] each, caller-owned,
 * overwritten).  {d_u[p], d_v[p]} runs over the unique undirected edges of
 * the cleaned input, each once.  No sync.
 */
TC_API tc_status tc_edge_list(const tc_graph* g, void* stream, int32_t* d_u, int32_t* d_v);

/*
 * T by one of the paper's surveyed kernels instead of
 * the grouped path, on the same oriented CSR, for the paper's comparison
 * on B200.  Writes T into device uint64 *d_count (no sync).
 *   TC_VARIANT_POLAK : edge-centric, one thread per oriented edge, sequential
 *                      merge of N+(u) and N+(v) (Fig. 3).
 *   TC_VARIANT_TRUST : vertex-centric, N+(u) hashed, 2-hop neighbours as
 *                      queries; d+(u) > 100 -> a 1024-thread block with 1024
 *                      buckets, 2..100 -> a warp with 32 buckets.
 * Errors: unknown variant or NULL pointer -> TC_ERR_INVALID_ARGUMENT.
 */
#define TC_VARIANT_POLAK 1
#define TC_VARIANT_TRUST 2
TC_API tc_status tc_count_variant(const tc_graph* g, int32_t variant, void* stream,
                                  uint64_t* d_count);

/*
 * Cost-balanced split of [0, m_live) into world_size contiguous ranges
 * (per-edge intersections are independent, and edge
 * chunks are the unit of work): h_bounds (host int64[world_size+1])
 * receives 0 = b_0 <= b_1 <= ... <= b_P = m_live, aligned to work chunks.
 * The cut points are binary-searched on a prefix of the plan's per-chunk
 * cost (a6: key lanes + seg_cost per edge + d+(v) and table words per group)
 * weighted by a time profile: the chunk list is cut into n_slices SLICES of
 * near-equal cost (tc_slice_bounds; for n_slices >= 2 slices never straddle
 * the class boundary) and slice i's cost units are weighted so that the whole slice
 * weighs h_ms[i].  Cut r is the chunk boundary nearest to r/P of the total.
 *   tc_partition          : the built-in profile - two slices (long class,
 *                           short class), a short-class unit weighing
 *                           TC_PARTITION_SHORT_RATIO long-class units.
 *   tc_partition_measured : h_ms from tc_calibrate (every rank must pass the
 *                           same profile, e.g. the ranks' average).
 * Host only.  Errors: NULL, world_size < 1, n_slices < 1, a negative or
 * non-finite h_ms entry -> TC_ERR_INVALID_ARGUMENT.
 */
#define TC_PARTITION_SHORT_RATIO 2.2 /* short vs long ns per cost unit (C3 2.21, C4 2.09) */
TC_API tc_status tc_partition(const tc_graph* g, int32_t world_size, int64_t* h_bounds);
TC_API tc_status tc_partition_measured(const tc_graph* g, int32_t world_size, int32_t n_slices,
                                       const double* h_ms, int64_t* h_bounds);

/*
 * Measure the time profile of the plan on this device: one warm-up count,
 * then every slice of tc_slice_bounds(n_slices) counted alone (one
 * tc_count_range call per slice, CUDA events on `stream`).  h_ms (host
 * double[n_slices]) receives the slices' ms (0 for an empty slice).
 * Synchronises.  Each slice is ~1/n_slices of a count, so it still fills the
 * GPU for n_slices up to a few hundred at configs C3/C4.
 */
TC_API tc_status tc_calibrate(const tc_graph* g, void* stream, int32_t n_slices, double* h_ms);

/*
 * Refine a profile for world_size ranks on this device: split by h_ms (as
 * tc_partition_measured), time every rank's range alone (one warm-up count,
 * then world_size tc_count_range calls, CUDA events on `stream`), and scale
 * each slice's h_ms (host double[n_slices], in place) by measured / predicted
 * time of the ranges it overlaps (cost-weighted).  The split of the refined
 * profile corrects what the slices mispredict, e.g. a range's launch tail
 * (C3 P = 8 with 256 slices: max/mean 1.115 -> 1.006).  Synchronises.  Every
 * rank must end with the same profile (average the refined ones).
 */
TC_API tc_status tc_refine_profile(const tc_graph* g, void* stream, int32_t world_size,
                                   int32_t n_slices, double* h_ms);

/*
 * Host only: the slices of a profile.  h_first (host int64[n_slices+1])
 * receives each slice's first CHUNK (h_first[n_slices] = n_chunks).  One
 * slice is the whole list; otherwise the long
 * class [0, n_long_chunks) gets round(n_slices * its cost share) slices (at
 * least 1 if non-empty, at most n_slices - 1 if the short class is
 * non-empty), the short class the rest; inside a class slice j starts at the
 * first chunk whose cost prefix reaches j/K of the class's cost.
 */
TC_API tc_status tc_slice_bounds(const int64_t* h_cost, int64_t n_chunks, int64_t n_long_chunks,
                                 int32_t n_slices, int64_t* h_first);

/*
 * Host-only form of the split (no GPU; CPU-tested): h_seg / h_cost (host
 * int64[n_chunks+1], non-decreasing) are the chunks' first edges and cost
 * prefix as tc_plan_chunks returns them, chunks [0, n_long_chunks) long;
 * h_ms the profile of tc_slice_bounds(n_slices).  Writes h_bounds as
 * tc_partition_measured does.
 */
TC_API tc_status tc_partition_chunks(const int64_t* h_seg, const int64_t* h_cost, int64_t n_chunks,
                                     int64_t n_long_chunks, int32_t n_slices, const double* h_ms,
                                     int32_t world_size, int64_t* h_bounds);

/*
 * The plan's work chunks, host copies: h_seg (host int64[n_chunks+1], or
 * NULL) receives each chunk's first live edge (h_seg[n_chunks] = m_live);
 * h_cost (host int64[n_chunks+1], or NULL) the plan cost prefix at those
 * edges (h_cost[n_long_chunks] = the long class's total).  Host only.
 */
TC_API tc_status tc_plan_chunks(const tc_graph* g, int64_t* h_seg, int64_t* h_cost);

/*
 * Host-only form of the same split (no GPU needed; tested on CPU):
 * given the exclusive cost prefix of `n_units` units (prefix[0] = 0,
 * prefix[n_units] = total, non-decreasing), writes the unit bounds that cut
 * the total cost into world_size near-equal contiguous parts.
 */
TC_API tc_status tc_partition_prefix(const int64_t* h_prefix, int64_t n_units, int32_t world_size,
                              int64_t* h_bounds);

/*
 * ------------------------------------------------------------------------
 * SHARDED preprocessing.  The same a1..a6 pipeline
 * split into stateless steps so that P ranks, each holding 1/P of the raw
 * pairs, build the identical replicated graph while the heavy sorts run on
 * 1/P of the keys each.  The exchange steps between them are collectives of
 * the caller (torch.distributed over NCCL; paper_conf_ipps_li0ptz24_b200.
 * sharded.build_csr_sharded drives them):
 *
 *   tc_shard_canon      a1 + a2 on the local pairs -> sorted unique keys
 *   tc_shard_histogram  per-bucket key counts (top bits)   -> all_reduce
 *   tc_shard_cuts       host: bucket cuts with near-equal key counts
 *   tc_shard_bounds     positions of the cuts in the local sorted keys
 *                                                            -> all_to_all
 *   tc_shard_unique     a2 (global dedup: equal keys meet on one rank) + a3
 *                       partial degrees                      -> all_reduce
 *   tc_rank_vertices    a4 (replicated: same degrees -> same ranking)
 *   tc_shard_orient     a5 relabel + orient + local sort
 *   (histogram / cuts / bounds again on the oriented keys)  -> all_to_all
 *   tc_sort_keys        local sort of the received row range
 *                       (rank r's slice precedes rank r+1's) -> all-gather
 *   tc_build_from_oriented  CSR + plan (a5, a6) from all m sorted keys
 *
 * KEY FORMAT: a key over a vertex bound n is (a << b) | c with a, c in
 * [0, n) and b = tc_key_bits(n) = max(1, ceil(log2 n)); canonical keys have
 * a < c (original ids), oriented keys a = rank u < c = rank v.
 * Keys are uint64 in device memory, caller-owned.  None of these calls keeps
 * state between calls; scratch is stream-ordered and freed before return.
 * ------------------------------------------------------------------------
 */

/* b = bits of one vertex field for a vertex bound n (n >= 0). */
TC_API int32_t tc_key_bits(int64_t n);

/*
 * a1 + a2 on one shard: canonical keys of the valid non-loop pairs of
 * (d_src, d_dst) (device int32[num_edges], caller-owned, unmodified), sorted
 * ascending and unique, into d_keys (device uint64, capacity >= num_edges;
 * may not alias the inputs).  *h_count = number written.  num_vertices >= 0
 * is REQUIRED (all ranks must agree on it).  Errors: id < 0 or >=
 * num_vertices -> TC_ERR_INVALID_ARGUMENT.  Synchronises.
 */
TC_API tc_status tc_shard_canon(const int32_t* d_src, const int32_t* d_dst, int64_t num_edges,
                                int64_t num_vertices, void* stream, uint64_t* d_keys,
                                int64_t* h_count);

/*
 * Key counts per bucket of the top `hist_bits` bits of the 2*tc_key_bits(n)
 * bit key space: d_hist[b] (device int64[2^hist_bits], overwritten) = number
 * of the `count` sorted keys whose bucket is b.  1 <= hist_bits <=
 * min(24, 2*tc_key_bits(n)).  Stream-ordered, no sync.
 */
TC_API tc_status tc_shard_histogram(const uint64_t* d_keys, int64_t count, int64_t n,
                                    int32_t hist_bits, void* stream, int64_t* d_hist);

/*
 * Host only: cut the buckets [0, n_buckets) into world_size contiguous
 * ranges of near-equal total count (h_hist: host int64[n_buckets], the
 * GLOBAL histogram).  h_cuts (host int64[world_size+1]) receives 0 = c_0 <=
 * ... <= c_P = n_buckets; rank r owns buckets [c_r, c_{r+1}).
 */
TC_API tc_status tc_shard_cuts(const int64_t* h_hist, int64_t n_buckets, int32_t world_size,
                               int64_t* h_cuts);

/*
 * Positions of the bucket cuts in `count` sorted keys: h_bounds (host
 * int64[world_size+1]) receives p_r = first key whose bucket >= c_r
 * (p_0 = 0, p_P = count), so keys [p_r, p_{r+1}) go to rank r.  Synchronises.
 */
TC_API tc_status tc_shard_bounds(const uint64_t* d_keys, int64_t count, int64_t n,
                                 int32_t hist_bits, const int64_t* h_cuts, int32_t world_size,
                                 void* stream, int64_t* h_bounds);

/*
 * a2 + a3 after the first exchange: sort d_keys[0, count) (canonical keys,
 * any order, device uint64, in place), drop duplicates (*h_count = unique
 * count, compacted to the front), and ADD each unique key's two endpoints to
 * d_degree (device int32[n], caller-zeroed; the all_reduce of the ranks'
 * arrays is the undirected degree).  Synchronises.
 */
TC_API tc_status tc_shard_unique(uint64_t* d_keys, int64_t count, int64_t n, void* stream,
                                 int64_t* h_count, int32_t* d_degree);

/*
 * a3 alone: ADD each of `count` keys' two endpoints to d_degree (device
 * int32[n], caller-zeroed).  For a single rank, whose tc_shard_canon output
 * is already globally sorted and unique.  Stream-ordered.
 */
TC_API tc_status tc_shard_degree(const uint64_t* d_keys, int64_t count, int64_t n, void* stream,
                                 int32_t* d_degree);

/*
 * a4: rank vertices by (degree ascending, id ascending), dropping
 * degree-0 vertices unless TC_KEEP_ISOLATED.  d_degree: device int32[n]
 * (global degrees).  Writes d_rank[v] (device int32[n]) for every kept v and
 * d_perm[r] = v (device int32, capacity n) for r < *h_n_active.  Identical
 * inputs give identical outputs on every rank.  Synchronises.
 */
TC_API tc_status tc_rank_vertices(const int32_t* d_degree, int64_t n, uint32_t flags,
                                  void* stream, int32_t* d_rank, int32_t* d_perm,
                                  int64_t* h_n_active);

/*
 * a5 (first half): relabel canonical keys (over n) to ranks and orient low
 * -> high rank: d_okeys[i] (device uint64[count], caller-owned, may
 * not alias d_keys) = (min(ra, rc) << tc_key_bits(n_active)) | max(ra, rc),
 * sorted ascending.  Stream-ordered.
 */
TC_API tc_status tc_shard_orient(const uint64_t* d_keys, int64_t count, int64_t n,
                                 const int32_t* d_rank, int64_t n_active, void* stream,
                                 uint64_t* d_okeys);

/* Sort count keys over vertex bound n (device uint64, in place).  Stream-ordered. */
TC_API tc_status tc_sort_keys(uint64_t* d_keys, int64_t count, int64_t n, void* stream);

/*
 * a5 (second half) + a6: a graph from ALL m oriented keys, globally sorted
 * and unique (device uint64[m] over n_active, caller-owned, unmodified), the
 * ranking's d_perm (device int32[n_active]; copied) and the original vertex
 * bound n_input.  Equal to what tc_build_csr builds from the union of the
 * shards (tests compare the CSR byte for byte).  Synchronises.
 */
TC_API tc_status tc_build_from_oriented(const uint64_t* d_okeys, int64_t m,
                                        const int32_t* d_perm, int64_t n_active,
                                        int64_t n_input, const tc_options* opts, void* stream,
                                        tc_graph** out);

/*
 * ------------------------------------------------------------------------
 * the cross-GPU sum of the partial counts done by
 * the library over NVLink peer memory (no NCCL).  This rank counts
 * [e_begin, e_end) (as tc_count_range) and the LAST CTA of its last count
 * launch (a grid-completion ticket) adds the partial into a SYMMETRIC buffer
 * on every rank and waits for every rank's contribution, so no extra launch
 * is made (a rank whose range is empty runs a one-thread finishing kernel):
 *   - d_mc != NULL: through an NVLS multicast address (one
 *     multimem.red.add.u64; the NVSwitch updates every replica);
 *   - else through the world unicast peer addresses h_peers[0..world) (one
 *     red.add.u64 per peer over NVLink P2P; h_peers[rank] == d_own).
 * d_own : this rank's unicast address of the buffer (device uint64[8]:
 *         words 0/1 = the sums of even / odd epochs, 2 = arrivals, 3 =
 *         POISON, 4 = the ticket; zero-initialised once, same layout on every
 *         rank; do not touch it between calls).  epoch: 1 for the first call
 *         on a buffer, +1 per call, equal on all ranks.  world <= TC_MAX_PEERS.
 * d_total (device uint64) receives T on every rank.  Stream-ordered; the
 * kernel spins until all ranks arrive, so every rank must make the call; if
 * some rank has not arrived within 20 s (TC_FUSED_TIMEOUT_MS) the kernel sets
 * the buffer's POISON word and writes UINT64_MAX to d_total instead of
 * hanging the stream; the buffer must then be recreated.
 * The multicast / peer mappings are the caller's plumbing (e.g. torch
 * symmetric memory); tc_mc_buffer_create makes a single-device one.
 */
#define TC_MAX_PEERS 16
TC_API tc_status tc_count_range_fused(const tc_graph* g, int64_t e_begin, int64_t e_end,
                                      uint64_t* d_own, uint64_t* d_mc, uint64_t* const* h_peers,
                                      int32_t world, uint64_t epoch, void* stream,
                                      uint64_t* d_total);

/*
 * A multicast object whose only member is the current device, its memory
 * mapped at a unicast (*d_uc) and a multicast (*d_mc) address, >= bytes,
 * zeroed.  For single-process use (tests, one-GPU runs of the f4 path);
 * TC_ERR_UNSUPPORTED where the device or driver has no multicast objects.
 * Synchronises the device.  Release with tc_mc_buffer_destroy.
 */
TC_API tc_status tc_mc_buffer_create(size_t bytes, void** handle, uint64_t** d_uc,
                                     uint64_t** d_mc);
TC_API void tc_mc_buffer_destroy(void* handle);

/* Release a graph (NULL is a no-op).  Waits on the host for the work the
 * stream-ordered entry points (tc_count_async, tc_count_range[_fused],
 * tc_count_variant, tc_support, tc_edge_list) enqueued on the graph, on
 * whatever stream, up to this call -- not for the whole device, so a build
 * running on another stream is not waited for -- then frees the graph's
 * buffers stream-ordered. */
TC_API void tc_free(tc_graph* g);

/*
 * Process-wide diagnostic counters of the count kernels on the current
 * device: h_counters (host uint64[4]) receives [0] = chunks whose two-choice
 * (cuckoo) table inserts failed and were rebuilt with linear probing
 * (reading C-24), [1..3] = 0 (reserved).  reset != 0 zeroes them
 * after reading.  Synchronises the device.
 */
TC_API tc_status tc_counters(uint64_t* h_counters, int32_t reset);

/*
 * Return the device memory the library keeps cached for reuse (its
 * stream-ordered pools keep freed blocks mapped so repeated builds do not
 * re-map memory) to the driver, for the current device.  Live graphs are
 * untouched.  Synchronises the device.
 */
TC_API tc_status tc_release_memory(void);

/* Thread-local text for the last non-OK status of this thread. */
TC_API const char* tc_last_error(void);

/* Library version string, e.g. "b200tc 0.1 sm_100a". */
TC_API const char* tc_version(void);

#ifdef __cplusplus
}
#endif
#endif /* TC_H */

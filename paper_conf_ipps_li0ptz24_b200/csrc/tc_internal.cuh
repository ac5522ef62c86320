// tc_internal.cuh — shared internals of libtc.so (not part of the C-ABI).
//
// Product path only: nothing here is shared with oracle/ (DESIGN.md §3).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <memory>
#include <mutex>
#include <string>
#include <utility>
#include <vector>

#include "tc.h"
#include "tc_fused.cuh"

namespace tc {

// ---------------------------------------------------------------- errors
struct Error {
  tc_status status;
  std::string msg;
};

[[noreturn]] void fail(tc_status s, const std::string& msg);
void check_cuda(cudaError_t e, const char* what, const char* file, int line);
#define TC_CUDA(x) ::tc::check_cuda((x), #x, __FILE__, __LINE__)
#define TC_LAUNCH() ::tc::check_cuda(cudaGetLastError(), "kernel launch", __FILE__, __LINE__)

// ---------------------------------------------------------------- memory
// Two stream-ordered pools: PERSISTENT buffers (the graph's CSR and plan,
// freed by tc_free) come from the device's default pool, build SCRATCH from a
// dedicated pool that only ever holds scratch.  Keeping them apart means the
// scratch pool is never fragmented by long-lived arrays, so once it has grown
// to a build's peak, identical builds reuse it without mapping new memory
// (mixed in one pool, builds next to a resident graph varied 110-420 ms).
void* dev_alloc(size_t bytes, cudaStream_t s, bool persistent);  // throws TC_ERR_OUT_OF_MEMORY
void dev_free(void* p, size_t bytes, cudaStream_t s);
void reserve_pool(size_t bytes, cudaStream_t s);  // grow the scratch pool once, up front
void trim_pools();  // tc_release_memory

// Owning device buffer (stream-ordered free on the stream it was made on).
template <class T>
struct DevBuf {
  T* p = nullptr;
  size_t n = 0;
  cudaStream_t s = nullptr;
  DevBuf() = default;
  DevBuf(size_t count, cudaStream_t st, bool persistent = false) : n(count), s(st) {
    if (count) p = static_cast<T*>(dev_alloc(count * sizeof(T), st, persistent));
  }
  DevBuf(const DevBuf&) = delete;
  DevBuf& operator=(const DevBuf&) = delete;
  DevBuf(DevBuf&& o) noexcept { swap(o); }
  DevBuf& operator=(DevBuf&& o) noexcept {
    reset();
    swap(o);
    return *this;
  }
  ~DevBuf() { reset(); }
  void swap(DevBuf& o) noexcept {
    std::swap(p, o.p);
    std::swap(n, o.n);
    std::swap(s, o.s);
  }
  void reset() {
    if (p) dev_free(p, n * sizeof(T), s);
    p = nullptr;
    n = 0;
  }
  T* get() const { return p; }
};

// ---------------------------------------------------------------- host trace
// TC_HOST_TRACE=1: host timestamps of a build's steps, one stderr line per
// build (diagnosing host-side delays of the host entry point).
bool host_trace_on();
void host_mark(const char* what);  // no-op unless TC_HOST_TRACE
void host_trace_flush();

// ---------------------------------------------------------------- options
struct Options {
  int chunk_cost = 16384;
  int seg_cost = 4;
  int huge_degree = 8192;
  int block_threads = 1024;
  int table_factor = 6;   // C3/C2/C5 sweep (r19o/r19p): 3 -> 6 with bitmap_factor 12: -7% / -18% / -23%
  int long_min = 32;
  bool long_min_auto = true;  // long_min not given: graphs under kSmallGraph edges are all short
  int probe_mode = 0;
  int bitmap_factor = 16;  // <= 0: never (r2p/r2q C3 k_count: 8 -> 42.9 ms, 12 -> 41.6, 16 -> 41.25, 32 -> 41.2)
};
Options resolve_options(const tc_options* o);

// ---------------------------------------------------------------- plan
// The dispatch plan.  Units:
//   segment s  = one LIVE oriented edge (u,v): its keys are the suffix of
//                N+(u) after v trimmed to [min N+(v), max N+(v)]
//                (keys outside cannot match), non-empty, stored as
//                col[seg_start[s] .. seg_start[s] + seg_len[s]).
//   class      = LONG (seg_len >= long_min: one warp walks the segment in
//                32-key tiles) or SHORT (keys of many segments flattened
//                over the lanes).  Segments [0, S_long) are long, [S_long,
//                S) short; inside a class they are ordered by (v, position).
//   group g    = one run of segments of one class with the same head v;
//                its table is N+(v) = col[row_ptr[v] .. row_ptr[v+1]).
//   work unit  = a key lane: a long segment has 32*ceil(len/32) (its tiles),
//                a short one len; key_prefix is their exclusive prefix.
//   chunk c    = segments [chunk_seg[c], chunk_seg[c+1]) of one class and
//                near-equal cost; chunks [0, n_long_chunks) are long.
struct PlanView {
  const int32_t* col;
  const uint32_t* key_prefix;  // [S+1] work-unit prefix mod 2^32 (chunk-relative differences < 2^32)
  const uint32_t* seg_start;   // [S] (col index; m < 2^32)
  const int32_t* seg_len;      // [S]
  const int32_t* seg_group;    // [S]
  const int64_t* ins_prefix;   // [G+1] prefix of d+(v)
  const int64_t* grp_ibase;    // [G]  = row_ptr[v] - ins_prefix[g]
  const int64_t* slot_prefix;  // [G+1] prefix of table words (0 for huge groups)
  const int32_t* grp_code;     // [G] table kind: n >= 2 hash slots, <= 0 bitmap (-base word)
  const int64_t* chunk_seg;    // [C+1]
  int64_t n_long_chunks;
  int probe_mode;
  int short_linear;            // short class always probes linearly (Tuning::short_linear)
  int max_kicks;               // cuckoo displacement bound (Tuning::max_kicks)
  int64_t m;                   // entries of col
  // support mode only (tc_support; nullptr when counting)
  const int64_t* seg_edge;     // [S] CSR position of segment s's own edge (u,v)
  unsigned* sup;               // [m] per-edge triangle counts (accumulated)
};

// SMEM a chunk needs (bytes): per segment staging + per group descriptor +
// hash slots.  Shared by the plan (sizing) and the kernel (layout).
// Layout of one chunk slot of the count kernel (tc_count.cu slot_view), all
// offsets from a 16-B aligned base: sT0..sT3 int32[round4(T)] each (long
// class: one descriptor per 32-key tile) | sB int64[S] | sGB int64[G] | sInfo
// int2[G] | sA int32[S+1] | sC int32[S] | sD int32[S] | sGP int32[G+1] | pad to
// 16 B | sHash int32[slots].
__host__ __device__ inline int64_t chunk_smem_bytes(int64_t S, int64_t G, int64_t slots,
                                                    int64_t T) {
  return 16 * ((T + 3) & ~int64_t(3)) + 20 * S + 20 * G + 8 + 16 + 4 * slots;
}

// Count-kernel launch tuning (not part of the C-ABI; TC_SLOTS, TC_GRAB_LONG,
// TC_GRAB_SHORT, TC_PROD_DIV, TC_WAIT_HINT, TC_CS_DIV, TC_SHORT_LINEAR,
// TC_CUCKOO_KICKS override
// the defaults for sweeps; every setting gives the same count).
struct Tuning {
  int slots = 3;          // chunk slots in SMEM (2..4)
  int grab_long = 0;      // tiles per consumer grab, long class (0 = static split)
  int grab_short = 0;     // keys per consumer grab, short class (0 = static split)
  int prod_div = 4;       // 1/prod_div of the warps are producers (r2h, C3 k_count: 5 -> 44.9 ms, 4 -> 42.9,
                          // 3 -> 44.3; C4: 629 / 583 / 576 ms)
  int wait_hint_ns = 0;   // mbarrier try_wait suspend hint (0 = none)
  int cs_div = 0;         // short-class chunk cost = chunk_cost / cs_div (0: auto, 2 when the live
                          // edges carry < 2 keys on average, e.g. road graphs, else 1)
  int short_linear = 1;   // short class: linear-probing tables (no cuckoo attempt)
  int prod_groups = 2;    // long class: producer groups filling slots concurrently (TC_PROD_GROUPS, 1..3;
                          // r2k: 1 -> 2 groups C3 k_count 42.8 -> 41.7 ms, C4 583 -> 544 ms)
  int batch = 0;          // long-class tiles per batch for block_threads <= 768 (TC_BATCH; see count_kernel)
  int max_kicks = 96;     // cuckoo displacements before a chunk rebuilds with linear probing (TC_CUCKOO_KICKS;
                          // 0 forces the rebuild of every chunk with a hash table: tests)
  int long_hash_dmax = 128;  // long-class candidates whose head gets a hash table with d+(v) <= this
                            // go to the short class (TC_LONG_HASH_DMAX; 0 = off; r4x/r4y/r5a: C3 step
                            // 44.4 -> 43.9 ms, C2 1.313 -> 1.283, C4 558 -> 555)
};
Tuning tuning_from_env();

// Bytes of plan metadata a count reads (the method's own bytes, DESIGN.md
// §6.2): per live edge its key_prefix / seg_start / seg_len / seg_group
// entries, per (chunk, group) visit the group's ins_prefix / slot_prefix /
// grp_ibase / grp_code entries, per chunk its two chunk_seg entries and the
// closing key_prefix / ins_prefix / slot_prefix entries.
constexpr int64_t kPlanEdgeBytes = 4 + 4 + 4 + 4;
constexpr int64_t kPlanGroupBytes = 8 + 8 + 8 + 4;
constexpr int64_t kPlanChunkBytes = 16 + 4 + 16;

struct Plan {
  Options opt;
  Tuning tune;
  int64_t S = 0, S_long = 0, G = 0, n_chunks = 0, n_long_chunks = 0, keys_total = 0;
  int64_t units_total = 0;
  DevBuf<uint32_t> key_prefix, seg_start;  // 32-bit: see PlanView
  DevBuf<int64_t> ins_prefix, grp_ibase, slot_prefix, chunk_seg;
  DevBuf<int32_t> seg_len, seg_group, grp_code;
  DevBuf<int64_t> chunk_cost;  // [n_chunks+1] plan cost prefix at each chunk's first edge
  // Host copies of chunk_seg / chunk_cost, made on first use (host_plan):
  // a count of the whole graph and a 1-rank partition never need them.
  mutable std::vector<int64_t> h_chunk_seg, h_chunk_cost;
  mutable std::shared_ptr<std::once_flag> host_once = std::make_shared<std::once_flag>();
  int64_t table_words = 0;   // sum over (chunk, group) visits of d+(v): table rows read per count
  int64_t group_visits = 0;  // (chunk, group) pairs
  uint64_t method_bytes = 0; // bytes one full count reads as designed (keys + plan + tables)
  uint64_t method_bytes_long = 0;  // the long class's share (its kernel, k_count)
  int64_t keys_long = 0;     // trimmed keys of the long class
  int64_t chunk_cost_long = 0, chunk_cost_short = 0;  // after SMEM-driven halving
  int64_t smem_bytes = 0;  // per chunk slot, long class (warp-specialised kernel)
  int64_t smem_flat = 0;   // per chunk, short class (flat kernel)
  int grid = 0, block = 0, grid_flat = 0;
};

}  // namespace tc

struct tc_graph {
  int64_t n_input = 0, n = 0, m = 0, max_out = 0;
  int bits = 1;  // bits of a vertex id in [0, n)
  tc::DevBuf<int64_t> row_ptr;
  tc::DevBuf<int32_t> col, perm;
  tc::DevBuf<int32_t> rowid;  // build scratch: row of every CSR position (a5 -> a6), then freed
  tc::Plan plan;
  uint64_t b_itc = 0;
  float ms[6] = {0, 0, 0, 0, 0, 0};
  // Streams that ran work reading this graph (the stream-ordered entry points
  // record an event after their launches): tc_free waits for these events
  // only, not for the whole device (a build on another stream runs on).
  struct Use {
    cudaStream_t s;
    cudaEvent_t ev;
  };
  mutable std::mutex use_mu;
  mutable std::vector<Use> uses;
};

namespace tc {

// The plan with its host chunk arrays present (copied from the device on
// first use; the graph's build has completed).  tc_api.cu.
const Plan& host_plan(const tc_graph* g);

// tc_build.cu
void build_graph(const int32_t* d_src, const int32_t* d_dst, int64_t m_gen, int64_t n,
                 uint32_t flags, const Options& opt, cudaStream_t s, tc_graph* g);
void build_plan(tc_graph* g, const Options& opt, cudaStream_t s);
void build_graph_host(const int32_t* h_src, const int32_t* h_dst, int64_t m_gen, int64_t n,
                      uint32_t flags, const Options& opt, cudaStream_t s, tc_graph* g);

// tc_build.cu, f2 sharded preprocessing (tc_shard_* in tc.h)
int key_bits(int64_t n);
int64_t shard_canon(const int32_t* d_src, const int32_t* d_dst, int64_t m_gen, int64_t n,
                    cudaStream_t s, uint64_t* out);
void shard_histogram(const uint64_t* keys, int64_t cnt, int64_t n, int hist_bits, cudaStream_t s,
                     int64_t* d_hist);
void shard_bounds(const uint64_t* keys, int64_t cnt, int64_t n, int hist_bits,
                  const int64_t* h_cuts, int P, cudaStream_t s, int64_t* h_bounds);
void sort_keys(uint64_t* keys, int64_t cnt, int64_t n, cudaStream_t s);
int64_t shard_unique(uint64_t* keys, int64_t cnt, int64_t n, cudaStream_t s, int32_t* d_deg);
void shard_degree(const uint64_t* keys, int64_t cnt, int64_t n, cudaStream_t s, int32_t* d_deg);
int64_t shard_rank(const int32_t* deg, int64_t n, uint32_t flags, cudaStream_t s, int32_t* rank,
                   int32_t* perm);
void shard_orient(const uint64_t* keys, int64_t cnt, int64_t n, const int32_t* rank,
                  int64_t n_act, cudaStream_t s, uint64_t* okeys);
void build_from_oriented(const uint64_t* okeys, int64_t m, const int32_t* perm, int64_t n_act,
                         int64_t n_input, const Options& opt, cudaStream_t s, tc_graph* g);

// tc_count.cu
// Returns the number of count kernels launched.  With `fuse` (f4), the last
// launch's last CTA adds the partial into the symmetric buffer of every rank
// and leaves T in *d_out; 0 launches = the caller must run fused_finish.
int count_chunks(const tc_graph* g, int64_t c_begin, int64_t c_end, int64_t e_begin,
                 int64_t e_end, cudaStream_t s, unsigned long long* d_out,
                 const FuseArgs* fuse = nullptr);
int count_occupancy(int block, int64_t smem_bytes, const Tuning& tu);  // CTAs per SM (0 = cannot launch)
int max_smem_per_block();
int max_chunk_smem(const Tuning& tu);  // SMEM one of the kernel's chunk slots may use
int max_flat_chunk_smem();      // SMEM one short-class chunk may use (3 CTAs per SM)
int flat_occupancy(int64_t smem_bytes);
int num_sms();
void support_all(const tc_graph* g, cudaStream_t s, unsigned* d_sup);   // f1, tc_support
void edge_ends(const tc_graph* g, cudaStream_t s, int32_t* d_u, int32_t* d_v);
void read_counters(uint64_t* h, bool reset);  // tc_counters

// tc_fused.cu (f4: fused cross-GPU sum over NVLink peer memory, tc_fused.cuh)
FuseArgs fuse_args(uint64_t* own, uint64_t* mc, uint64_t* const* peers, int world,
                   uint64_t epoch);
void fused_finish(unsigned long long* d_total, const FuseArgs& f, cudaStream_t s);
void* mc_create(size_t bytes, uint64_t** uc, uint64_t** mc);
void mc_destroy(void* h);

// tc_variants.cu (f3: the paper's Polak / TRUST kernels on this CSR)
void count_variant(const tc_graph* g, int variant, cudaStream_t s, unsigned long long* d_out);

}  // namespace tc

// tc_api.cu — the C-ABI boundary (include/tc.h).  Argument checking, error
// translation (no exception crosses the ABI), the allocator hook, and the
// host-side range/partition logic.  SURVEY.md §8(b).
#include <algorithm>
#include <atomic>
#include <chrono>
#include <cmath>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <new>
#include <vector>

#include <mutex>

#include "tc_internal.cuh"

namespace {
thread_local std::string t_last_error;

tc_alloc_fn g_alloc = nullptr;
tc_free_fn g_free = nullptr;
void* g_ctx = nullptr;

template <class F>
tc_status guarded(F f) {
  try {
    f();
    return TC_OK;
  } catch (const tc::Error& e) {
    t_last_error = e.msg;
    return e.status;
  } catch (const std::bad_alloc&) {
    t_last_error = "host allocation failed";
    return TC_ERR_OUT_OF_MEMORY;
  } catch (...) {
    t_last_error = "unexpected internal error";
    return TC_ERR_CUDA;
  }
}

void require(bool ok, const char* msg) {
  if (!ok) tc::fail(TC_ERR_INVALID_ARGUMENT, msg);
}

}  // namespace

namespace tc {

void fail(tc_status s, const std::string& msg) { throw Error{s, msg}; }

void check_cuda(cudaError_t e, const char* what, const char* file, int line) {
  if (e == cudaSuccess) return;
  if (e == cudaErrorMemoryAllocation) {
    cudaGetLastError();
    fail(TC_ERR_OUT_OF_MEMORY, std::string("CUDA out of memory in ") + what);
  }
  char buf[512];
  snprintf(buf, sizeof(buf), "%s: %s (%s:%d)", what, cudaGetErrorString(e), file, line);
  fail(TC_ERR_CUDA, buf);
}

bool host_trace_on() {
  static const bool on = std::getenv("TC_HOST_TRACE") != nullptr;
  return on;
}
namespace {
thread_local std::vector<std::pair<const char*, std::chrono::steady_clock::time_point>> g_marks;
}
void host_mark(const char* what) {
  if (host_trace_on()) g_marks.emplace_back(what, std::chrono::steady_clock::now());
}
void host_trace_flush() {
  if (!host_trace_on() || g_marks.empty()) return;
  std::string line = "[tc host]";
  for (size_t i = 1; i < g_marks.size(); ++i) {
    char b[96];
    snprintf(b, sizeof(b), " %s %.2f", g_marks[i].first,
             std::chrono::duration<double, std::milli>(g_marks[i].second - g_marks[i - 1].second).count());
    line += b;
  }
  fprintf(stderr, "%s\n", line.c_str());
  g_marks.clear();
}

namespace {
constexpr int kMaxDevices = 64;

// Release threshold "never": freed blocks stay mapped across syncs (without
// this every build re-maps its scratch, tens of ms at config C2).  (Turning
// off the pools' internal cross-stream reuse dependencies made the host
// entry's steps vary, C5 13 -> 13-119 ms, profiles/r5c_e2e.txt; kept on.)
void keep_mapped(cudaMemPool_t pool) {
  uint64_t thr = UINT64_MAX;
  cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
}

// The device's default pool (persistent buffers) or the library's own scratch
// pool, created on first use.  nullptr if the device cannot be queried.
cudaMemPool_t pool_of(bool persistent) {
  static cudaMemPool_t scratch[kMaxDevices] = {};
  static bool default_ready[kMaxDevices] = {};
  static std::mutex mu;  // first use may come from several host threads
  std::lock_guard<std::mutex> lk(mu);
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) {
    cudaGetLastError();
    return nullptr;
  }
  if (persistent) {
    cudaMemPool_t p = nullptr;
    if (cudaDeviceGetDefaultMemPool(&p, dev) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
    if (!default_ready[dev]) {
      keep_mapped(p);
      default_ready[dev] = true;
    }
    return p;
  }
  if (!scratch[dev]) {
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.handleTypes = cudaMemHandleTypeNone;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    if (cudaMemPoolCreate(&scratch[dev], &props) != cudaSuccess) {
      cudaGetLastError();
      scratch[dev] = nullptr;
      return nullptr;
    }
    keep_mapped(scratch[dev]);
  }
  return scratch[dev];
}
}  // namespace

void* dev_alloc(size_t bytes, cudaStream_t s, bool persistent) {
  void* p = nullptr;
  if (g_alloc) {
    p = g_alloc(bytes, (void*)s, g_ctx);
    if (!p) fail(TC_ERR_OUT_OF_MEMORY, "allocator hook returned NULL");
    return p;
  }
  cudaMemPool_t pool = pool_of(persistent);
  cudaError_t e = pool ? cudaMallocFromPoolAsync(&p, bytes, pool, s) : cudaMallocAsync(&p, bytes, s);
  if (e != cudaSuccess || !p) {
    cudaGetLastError();
    fail(TC_ERR_OUT_OF_MEMORY, "cudaMallocAsync failed (" + std::to_string(bytes) + " bytes)");
  }
  return p;
}

// Grow the scratch pool in one step so that a build's scratch allocations
// reuse already-mapped memory: mapping physical memory inside the build
// (pool growth on demand) made identical builds vary by 3-10x in time.
// The scratch pool only ever grows (release threshold "never"; trim_pools
// resets it), and nothing holds scratch between builds, so once it has been
// grown to `bytes` a later build of at most that size skips the driver
// queries: they cost 0.1-9 ms per build of the host entry at C2 and made its
// steps vary (TC_HOST_TRACE, profiles/r5m_*).
std::atomic<uint64_t> g_reserved_hint[64];

void reserve_pool(size_t bytes, cudaStream_t s) {
  if (g_alloc || bytes == 0) return;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) {
    cudaGetLastError();
    return;
  }
  if ((uint64_t)bytes <= g_reserved_hint[dev].load(std::memory_order_relaxed)) return;
  cudaMemPool_t pool = pool_of(false);
  if (!pool) return;
  uint64_t reserved = 0, used = 0;
  cudaMemPoolGetAttribute(pool, cudaMemPoolAttrReservedMemCurrent, &reserved);
  cudaMemPoolGetAttribute(pool, cudaMemPoolAttrUsedMemCurrent, &used);
  if (reserved - used >= bytes) {
    if (used == 0) g_reserved_hint[dev].store(reserved, std::memory_order_relaxed);
    return;
  }
  size_t free_b = 0, total_b = 0;
  cudaMemGetInfo(&free_b, &total_b);
  const size_t want = bytes - (size_t)(reserved - used);
  const size_t cap = free_b > (size_t(4) << 30) ? free_b - (size_t(4) << 30) : 0;
  const size_t grow = want < cap ? want : cap;
  if (grow == 0) return;
  void* p = nullptr;
  if (cudaMallocFromPoolAsync(&p, grow, pool, s) == cudaSuccess && p) {
    cudaFreeAsync(p, s);
    if (used == 0) g_reserved_hint[dev].store(reserved + grow, std::memory_order_relaxed);
  }
  cudaGetLastError();
}

// Give the pools' cached (freed but still mapped) memory of the current
// device back to the driver: tc_release_memory.
void trim_pools() {
  TC_CUDA(cudaDeviceSynchronize());
  for (auto& h : g_reserved_hint) h.store(0, std::memory_order_relaxed);
  for (bool persistent : {false, true}) {
    cudaMemPool_t pool = pool_of(persistent);
    if (pool) TC_CUDA(cudaMemPoolTrimTo(pool, 0));
  }
}

const Plan& host_plan(const tc_graph* g) {
  const Plan& P = g->plan;
  std::call_once(*P.host_once, [&] {
    std::vector<int64_t> seg(P.n_chunks + 1), cost(P.n_chunks + 1);
    TC_CUDA(cudaMemcpy(seg.data(), P.chunk_seg.get(), sizeof(int64_t) * seg.size(),
                       cudaMemcpyDeviceToHost));
    TC_CUDA(cudaMemcpy(cost.data(), P.chunk_cost.get(), sizeof(int64_t) * cost.size(),
                       cudaMemcpyDeviceToHost));
    P.h_chunk_seg.swap(seg);
    P.h_chunk_cost.swap(cost);
  });
  return P;
}

void dev_free(void* p, size_t bytes, cudaStream_t s) {
  if (!p) return;
  if (g_free) {
    g_free(p, bytes, (void*)s, g_ctx);
    return;
  }
  cudaFreeAsync(p, s);
}

Options resolve_options(const tc_options* o) {
  Options r;
  if (!o) return r;
  if (o->chunk_cost) r.chunk_cost = o->chunk_cost;
  if (o->seg_cost) r.seg_cost = o->seg_cost;
  if (o->huge_degree) r.huge_degree = o->huge_degree;
  if (o->block_threads) r.block_threads = o->block_threads;
  if (o->table_factor) r.table_factor = o->table_factor;
  if (o->long_min) {
    r.long_min = o->long_min;
    r.long_min_auto = false;
  }
  if (o->probe_mode) r.probe_mode = o->probe_mode;
  if (o->bitmap_factor) r.bitmap_factor = o->bitmap_factor;
  require(r.chunk_cost >= 64, "chunk_cost must be >= 64");
  require(r.seg_cost >= 1, "seg_cost must be >= 1");
  require(r.huge_degree >= 1, "huge_degree must be >= 1");
  require(r.block_threads >= 64 && r.block_threads <= 1024 && r.block_threads % 32 == 0,
          "block_threads must be a multiple of 32 in [64, 1024]");
  require(r.table_factor >= 2 && r.table_factor <= 16, "table_factor must be in [2, 16]");
  require(r.long_min >= 1, "long_min must be >= 1");
  require(r.probe_mode == 0 || r.probe_mode == 1, "probe_mode must be 0 or 1");
  return r;
}

}  // namespace tc

namespace {

// Rebinds every stream-ordered buffer of the graph to `s` so frees are
// ordered after the work that used them.
// Record that work reading g was enqueued on s (tc_free waits for it).
void note_use(const tc_graph* g, void* stream) {
  const cudaStream_t s = (cudaStream_t)stream;
  std::lock_guard<std::mutex> lk(g->use_mu);
  for (auto& u : g->uses)
    if (u.s == s) {
      TC_CUDA(cudaEventRecord(u.ev, s));
      return;
    }
  tc_graph::Use u{s, nullptr};
  TC_CUDA(cudaEventCreateWithFlags(&u.ev, cudaEventDisableTiming));
  g->uses.push_back(u);
  TC_CUDA(cudaEventRecord(u.ev, s));
}

void rebind(tc_graph* g, cudaStream_t s) {
  g->row_ptr.s = g->col.s = g->perm.s = s;
  tc::Plan& P = g->plan;
  P.key_prefix.s = P.seg_start.s = s;
  P.ins_prefix.s = P.grp_ibase.s = P.slot_prefix.s = P.chunk_seg.s = P.chunk_cost.s = s;
  P.seg_len.s = P.seg_group.s = P.grp_code.s = s;
}

// Chunks overlapping the live edges [e_begin, e_end): the first whose end is
// > e_begin up to the last whose start is < e_end.
void chunk_range(const tc_graph* g, int64_t e_begin, int64_t e_end, int64_t* c_begin,
                 int64_t* c_end) {
  *c_begin = *c_end = 0;
  if (e_end <= e_begin) return;
  if (e_begin == 0 && e_end == g->plan.S) {  // the whole graph: no host chunk arrays needed
    *c_end = g->plan.n_chunks;
    return;
  }
  const tc::Plan& P = tc::host_plan(g);
  const auto& cs = P.h_chunk_seg;
  *c_begin = std::max<int64_t>(std::upper_bound(cs.begin(), cs.end(), e_begin) - cs.begin() - 1, 0);
  *c_end = std::min<int64_t>(std::lower_bound(cs.begin(), cs.end(), e_end) - cs.begin(), P.n_chunks);
}

tc_status build_impl(const int32_t* src, const int32_t* dst, int64_t num_edges,
                     int64_t num_vertices, uint32_t flags, const tc_options* opts, void* stream,
                     tc_graph** out, bool host) {
  if (out) *out = nullptr;
  tc_graph* g = nullptr;
  tc_status st = guarded([&] {
    require(out != nullptr, "out is NULL");
    require(num_edges >= 0, "num_edges < 0");
    require(num_edges == 0 || (src && dst), "src/dst is NULL");
    require(num_vertices >= -1 && num_vertices <= 0x7fffffffLL,
            "num_vertices must be -1 or in [0, 2^31-1]");
    require((flags & ~TC_KEEP_ISOLATED) == 0, "unknown flag bits");
    const tc::Options opt = tc::resolve_options(opts);
    cudaStream_t s = (cudaStream_t)stream;
    // peak scratch of a1..a6 is ~72 B per input pair (sort double buffers,
    // plan arrays) + ~48 B per vertex; the host entry adds the 8-B pair copy
    const int64_t nv = num_vertices > 0 ? num_vertices : 0;
    // + the a2 hash set (u64, capacity the power of two >= 2 num_edges)
    size_t cap = 1024;
    while ((int64_t)cap < 2 * num_edges && num_edges <= (int64_t(1) << 25)) cap <<= 1;
    tc::host_mark("start");
    tc::reserve_pool((size_t)num_edges * (host ? 80 : 72) + (size_t)nv * 48 + cap * 8, s);
    tc::host_mark("reserve_pool");
    g = new tc_graph();
    if (host) {
      tc::build_graph_host(src, dst, num_edges, num_vertices, flags, opt, s, g);
    } else {
      tc::build_graph(src, dst, num_edges, num_vertices, flags, opt, s, g);
    }
    tc::host_mark("return");
    tc::host_trace_flush();
  });
  if (st != TC_OK) {
    if (g) {
      cudaStreamSynchronize((cudaStream_t)stream);
      delete g;
    }
    return st;
  }
  *out = g;
  return TC_OK;
}

}  // namespace

extern "C" {

tc_status tc_set_allocator(tc_alloc_fn alloc, tc_free_fn free_fn, void* ctx) {
  if ((alloc == nullptr) != (free_fn == nullptr)) {
    t_last_error = "alloc and free hooks must both be set or both be NULL";
    return TC_ERR_INVALID_ARGUMENT;
  }
  g_alloc = alloc;
  g_free = free_fn;
  g_ctx = ctx;
  return TC_OK;
}

tc_status tc_build_csr(const int32_t* d_src, const int32_t* d_dst, int64_t num_edges,
                       int64_t num_vertices, uint32_t flags, const tc_options* opts,
                       void* stream, tc_graph** out) {
  return build_impl(d_src, d_dst, num_edges, num_vertices, flags, opts, stream, out, false);
}

tc_status tc_build_csr_host(const int32_t* h_src, const int32_t* h_dst, int64_t num_edges,
                            int64_t num_vertices, uint32_t flags, const tc_options* opts,
                            void* stream, tc_graph** out) {
  return build_impl(h_src, h_dst, num_edges, num_vertices, flags, opts, stream, out, true);
}

tc_status tc_replan(tc_graph* g, const tc_options* opts, void* stream) {
  return guarded([&] {
    require(g != nullptr, "graph is NULL");
    const tc::Options opt = tc::resolve_options(opts);
    cudaStream_t s = (cudaStream_t)stream;
    TC_CUDA(cudaStreamSynchronize(s));
    rebind(g, s);
    tc::build_plan(g, opt, s);
    TC_CUDA(cudaStreamSynchronize(s));
  });
}

tc_status tc_graph_info(const tc_graph* g, tc_graph_info_t* o) {
  return guarded([&] {
    require(g && o, "NULL argument");
    std::memset(o, 0, sizeof(*o));
    const tc::Plan& P = g->plan;
    o->n_input = g->n_input;
    o->n = g->n;
    o->m = g->m;
    o->max_out_degree = g->max_out;
    o->m_live = P.S;
    o->n_groups = P.G;
    o->n_chunks = P.n_chunks;
    o->keys_total = P.keys_total;
    o->b_itc = g->b_itc;
    o->smem_bytes = P.smem_bytes;
    o->count_grid = P.grid;
    o->count_block = P.block;
    o->row_ptr = g->row_ptr.get();
    o->col = g->col.get();
    o->perm = g->perm.get();
    o->ms_canon = g->ms[0];
    o->ms_sort_unique = g->ms[1];
    o->ms_degree_rank = g->ms[2];
    o->ms_orient_csr = g->ms[3];
    o->ms_plan = g->ms[4];
    o->ms_total = g->ms[5];
    o->n_long_chunks = P.n_long_chunks;
    o->method_bytes = P.method_bytes;
    o->table_words = P.table_words;
    o->group_visits = P.group_visits;
    o->m_live_long = P.S_long;
    o->method_bytes_long = P.method_bytes_long;
    o->keys_long = P.keys_long;
  });
}

tc_status tc_count_async(const tc_graph* g, void* stream, uint64_t* d_count) {
  return guarded([&] {
    require(g && d_count, "NULL argument");
    tc::count_chunks(g, 0, g->plan.n_chunks, 0, g->plan.S, (cudaStream_t)stream,
                     reinterpret_cast<unsigned long long*>(d_count));
    note_use(g, stream);
  });
}

tc_status tc_count(const tc_graph* g, void* stream, uint64_t* h_count) {
  return guarded([&] {
    require(g && h_count, "NULL argument");
    cudaStream_t s = (cudaStream_t)stream;
    // The 8-B result: a per-thread device word (no pool allocation, so no
    // reuse dependency on another stream's frees) copied into per-thread
    // pinned memory (a copy into pageable stack memory held a build's H2D
    // copies on another stream back until this count finished: C3 pipelined
    // e2e 124 vs 100 ms per step, profiles/r4o_pipeline_variants.txt).  The
    // call is synchronous, so one word per thread and device suffices.
    thread_local struct Result {
      int dev = -1;
      unsigned long long* d = nullptr;
      unsigned long long* h = nullptr;
      ~Result() {
        if (d) cudaFree(d);
        if (h) cudaFreeHost(h);
      }
    } res;
    int dev = 0;
    TC_CUDA(cudaGetDevice(&dev));
    if (res.dev != dev) {
      if (res.d) cudaFree(res.d);
      res.d = nullptr;
      TC_CUDA(cudaMalloc(&res.d, sizeof(unsigned long long)));
      res.dev = dev;
    }
    if (!res.h) TC_CUDA(cudaMallocHost(&res.h, sizeof(unsigned long long)));
    tc::count_chunks(g, 0, g->plan.n_chunks, 0, g->plan.S, s, res.d);
    TC_CUDA(cudaMemcpyAsync(res.h, res.d, sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
    TC_CUDA(cudaStreamSynchronize(s));
    *h_count = *res.h;
  });
}

tc_status tc_count_range(const tc_graph* g, int64_t e_begin, int64_t e_end, void* stream,
                         uint64_t* d_partial) {
  return guarded([&] {
    require(g && d_partial, "NULL argument");
    const tc::Plan& P = g->plan;
    require(0 <= e_begin && e_begin <= e_end && e_end <= P.S,
            "need 0 <= e_begin <= e_end <= m_live");
    int64_t c_begin = 0, c_end = 0;
    chunk_range(g, e_begin, e_end, &c_begin, &c_end);
    tc::count_chunks(g, c_begin, c_end, e_begin, e_end, (cudaStream_t)stream,
                     reinterpret_cast<unsigned long long*>(d_partial));
    note_use(g, stream);
  });
}

tc_status tc_count_range_fused(const tc_graph* g, int64_t e_begin, int64_t e_end, uint64_t* d_own,
                               uint64_t* d_mc, uint64_t* const* h_peers, int32_t world,
                               uint64_t epoch, void* stream, uint64_t* d_total) {
  return guarded([&] {
    require(g && d_total && d_own, "NULL argument");
    require(world >= 1 && world <= TC_MAX_PEERS, "world must be in [1, TC_MAX_PEERS]");
    require(epoch >= 1, "epoch must be >= 1");
    require(d_mc || h_peers, "need a multicast address or the peer addresses");
    require(0 <= e_begin && e_begin <= e_end && e_end <= g->plan.S,
            "need 0 <= e_begin <= e_end <= m_live");
    if (!d_mc)
      for (int r = 0; r < world; ++r) require(h_peers[r] != nullptr, "NULL peer address");
    const tc::FuseArgs f = tc::fuse_args(d_own, d_mc, h_peers, world, epoch);
    int64_t c_begin = 0, c_end = 0;
    chunk_range(g, e_begin, e_end, &c_begin, &c_end);
    // the count kernel's last CTA runs the cross-rank sum; a rank whose range
    // launches no kernel still takes part through the finishing kernel
    unsigned long long* tot = reinterpret_cast<unsigned long long*>(d_total);
    if (tc::count_chunks(g, c_begin, c_end, e_begin, e_end, (cudaStream_t)stream, tot, &f) == 0)
      tc::fused_finish(tot, f, (cudaStream_t)stream);
    note_use(g, stream);
  });
}

tc_status tc_mc_buffer_create(size_t bytes, void** handle, uint64_t** d_uc, uint64_t** d_mc) {
  if (handle) *handle = nullptr;
  return guarded([&] {
    require(handle && d_uc && d_mc, "NULL argument");
    require(bytes > 0, "bytes must be > 0");
    *handle = tc::mc_create(bytes, d_uc, d_mc);
  });
}

void tc_mc_buffer_destroy(void* handle) { tc::mc_destroy(handle); }

tc_status tc_count_variant(const tc_graph* g, int32_t variant, void* stream, uint64_t* d_count) {
  return guarded([&] {
    require(g && d_count, "NULL argument");
    require(variant == TC_VARIANT_POLAK || variant == TC_VARIANT_TRUST, "unknown variant");
    tc::count_variant(g, variant, (cudaStream_t)stream,
                      reinterpret_cast<unsigned long long*>(d_count));
    note_use(g, stream);
  });
}

tc_status tc_support(const tc_graph* g, void* stream, uint32_t* d_support) {
  return guarded([&] {
    require(g != nullptr, "graph is NULL");
    require(g->m == 0 || d_support != nullptr, "d_support is NULL");
    tc::support_all(g, (cudaStream_t)stream, reinterpret_cast<unsigned*>(d_support));
    note_use(g, stream);
  });
}

tc_status tc_edge_list(const tc_graph* g, void* stream, int32_t* d_u, int32_t* d_v) {
  return guarded([&] {
    require(g != nullptr, "graph is NULL");
    require(g->m == 0 || (d_u && d_v), "d_u/d_v is NULL");
    tc::edge_ends(g, (cudaStream_t)stream, d_u, d_v);
    note_use(g, stream);
  });
}

tc_status tc_partition_prefix(const int64_t* h_prefix, int64_t n_units, int32_t world_size,
                              int64_t* h_bounds) {
  return guarded([&] {
    require(h_prefix && h_bounds, "NULL argument");
    require(n_units >= 0, "n_units < 0");
    require(world_size >= 1, "world_size < 1");
    const int64_t total = h_prefix[n_units];
    h_bounds[0] = 0;
    for (int32_t r = 1; r < world_size; ++r) {
      // first unit whose exclusive prefix reaches r/world of the total cost
      const long double t = (long double)total * r / world_size;
      const int64_t* it = std::lower_bound(h_prefix, h_prefix + n_units + 1, t,
                                           [](int64_t a, long double b) { return (long double)a < b; });
      int64_t b = it - h_prefix;
      b = std::min(std::max(b, h_bounds[r - 1]), n_units);
      h_bounds[r] = b;
    }
    h_bounds[world_size] = n_units;
  });
}

namespace {

// Slice bounds (chunk indices) of an n_slices profile: tc_slice_bounds.
void slice_bounds(const int64_t* cost, int64_t nc, int64_t nL, int32_t K, int64_t* first) {
  if (K == 1) {  // one slice: the whole chunk list
    first[0] = 0;
    first[1] = nc;
    return;
  }
  const long double total = (long double)cost[nc], cl = (long double)cost[nL];
  int KL = 0;
  if (nL > 0) {
    KL = total > 0 ? (int)std::llround((long double)K * cl / total) : K;
    KL = std::max(KL, 1);
    if (nc > nL) KL = std::min(KL, K - 1);
    KL = std::min(KL, K);
  }
  const int KS = K - KL;
  auto fill = [&](int64_t c0, int64_t c1, int k, int64_t* out) {
    // out[j] = first chunk in [c0, c1] whose cost prefix reaches j/k of the class
    const long double base = (long double)cost[c0], span = (long double)cost[c1] - base;
    for (int j = 0; j < k; ++j) {
      const long double t = base + span * j / k;
      int64_t lo = c0, hi = c1;
      while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if ((long double)cost[mid] < t) lo = mid + 1; else hi = mid;
      }
      out[j] = j == 0 ? c0 : lo;
    }
  };
  if (KL > 0) fill(0, nL, KL, first);
  if (KS > 0) fill(nL, nc, KS, first + KL);
  first[K] = nc;
  for (int j = 1; j <= K; ++j) first[j] = std::max(first[j], first[j - 1]);
}

}  // namespace

tc_status tc_slice_bounds(const int64_t* h_cost, int64_t n_chunks, int64_t n_long_chunks,
                          int32_t n_slices, int64_t* h_first) {
  return guarded([&] {
    require(h_cost && h_first, "NULL argument");
    require(n_chunks >= 0 && n_long_chunks >= 0 && n_long_chunks <= n_chunks, "bad chunk counts");
    require(n_slices >= 1, "n_slices < 1");
    for (int64_t c = 0; c < n_chunks; ++c) require(h_cost[c] <= h_cost[c + 1], "cost must be non-decreasing");
    slice_bounds(h_cost, n_chunks, n_long_chunks, n_slices, h_first);
  });
}

namespace {

// The profile's time up to every chunk boundary c (W[c], c in [0, nc]):
// slice i contributes h_ms[i] spread over its chunks in proportion to their
// plan cost (a slice without cost weighs its ms at its first boundary).
// Non-decreasing.  `first` receives the slice bounds.
std::vector<long double> profile_prefix(const int64_t* cost, int64_t nc, int64_t nL, int32_t K,
                                        const double* ms, std::vector<int64_t>& first) {
  first.assign(K + 1, 0);
  slice_bounds(cost, nc, nL, K, first.data());
  std::vector<long double> W(nc + 1, 0);
  long double acc = 0;
  for (int32_t i = 0; i < K; ++i) {
    const int64_t a = first[i], b = first[i + 1];
    const long double c0 = (long double)cost[a], span = (long double)cost[b] - c0;
    for (int64_t c = a; c < b; ++c)
      W[c] = acc + (span > 0 ? ((long double)cost[c] - c0) / span : 0) * (long double)ms[i];
    acc += (long double)ms[i];
  }
  W[nc] = acc;
  return W;
}

// Chunk-boundary cuts of W into P parts (nearest boundary to r/P of the total).
std::vector<int64_t> cut_chunks(const std::vector<long double>& W, int32_t P) {
  const int64_t nc = (int64_t)W.size() - 1;
  std::vector<int64_t> cb(P + 1, 0);
  cb[P] = nc;
  int64_t prev = 0;
  for (int32_t r = 1; r < P; ++r) {
    const long double t = W[nc] * r / P;
    int64_t lo = std::lower_bound(W.begin() + prev, W.end(), t) - W.begin();
    if (lo > prev && t - W[lo - 1] < W[lo] - t) --lo;  // the nearer boundary
    cb[r] = prev = lo;
  }
  return cb;
}

void check_profile_args(const int64_t* h_seg, const int64_t* h_cost, int64_t n_chunks,
                        int64_t n_long_chunks, int32_t n_slices, const double* h_ms,
                        int32_t world_size) {
  require(h_seg && h_cost && h_ms, "NULL argument");
  require(n_chunks >= 0 && n_long_chunks >= 0 && n_long_chunks <= n_chunks, "bad chunk counts");
  require(world_size >= 1, "world_size < 1");
  require(n_slices >= 1, "n_slices < 1");
  for (int32_t i = 0; i < n_slices; ++i)
    require(std::isfinite(h_ms[i]) && h_ms[i] >= 0, "profile entries must be finite and >= 0");
  for (int64_t c = 0; c < n_chunks; ++c)
    require(h_seg[c] <= h_seg[c + 1] && h_cost[c] <= h_cost[c + 1], "prefixes must be non-decreasing");
}

}  // namespace

tc_status tc_partition_chunks(const int64_t* h_seg, const int64_t* h_cost, int64_t n_chunks,
                              int64_t n_long_chunks, int32_t n_slices, const double* h_ms,
                              int32_t world_size, int64_t* h_bounds) {
  return guarded([&] {
    require(h_bounds != nullptr, "NULL argument");
    check_profile_args(h_seg, h_cost, n_chunks, n_long_chunks, n_slices, h_ms, world_size);
    std::vector<int64_t> first;
    const auto W = profile_prefix(h_cost, n_chunks, n_long_chunks, n_slices, h_ms, first);
    const auto cb = cut_chunks(W, world_size);
    for (int32_t r = 0; r <= world_size; ++r) h_bounds[r] = h_seg[cb[r]];
  });
}

tc_status tc_refine_profile(const tc_graph* g, void* stream, int32_t world_size, int32_t n_slices,
                            double* h_ms) {
  return guarded([&] {
    require(g && h_ms, "NULL argument");
    const tc::Plan& P = tc::host_plan(g);
    check_profile_args(P.h_chunk_seg.data(), P.h_chunk_cost.data(), P.n_chunks, P.n_long_chunks,
                       n_slices, h_ms, world_size);
    if (P.n_chunks == 0 || world_size == 1) return;
    cudaStream_t s = (cudaStream_t)stream;
    std::vector<int64_t> first;
    const auto W = profile_prefix(P.h_chunk_cost.data(), P.n_chunks, P.n_long_chunks, n_slices, h_ms,
                                  first);
    const auto cb = cut_chunks(W, world_size);
    // time every range alone, as its rank would count it
    tc::DevBuf<unsigned long long> d(1, s);
    std::vector<cudaEvent_t> ev(world_size + 1, nullptr);
    struct Guard {
      std::vector<cudaEvent_t>& e;
      ~Guard() {
        for (auto x : e)
          if (x) cudaEventDestroy(x);
      }
    } guard{ev};
    for (auto& e : ev) TC_CUDA(cudaEventCreate(&e));
    tc::count_chunks(g, 0, P.n_chunks, 0, P.S, s, d.get());  // warm-up
    TC_CUDA(cudaEventRecord(ev[0], s));
    for (int32_t r = 0; r < world_size; ++r) {
      if (cb[r + 1] > cb[r])
        tc::count_chunks(g, cb[r], cb[r + 1], P.h_chunk_seg[cb[r]], P.h_chunk_seg[cb[r + 1]], s,
                         d.get());
      TC_CUDA(cudaEventRecord(ev[r + 1], s));
    }
    TC_CUDA(cudaEventSynchronize(ev[world_size]));
    std::vector<double> f(world_size, 1.0);
    for (int32_t r = 0; r < world_size; ++r) {
      float ms = 0;
      TC_CUDA(cudaEventElapsedTime(&ms, ev[r], ev[r + 1]));
      const long double pred = W[cb[r + 1]] - W[cb[r]];
      if (cb[r + 1] > cb[r] && pred > 0) f[r] = (double)(ms / pred);
    }
    // slice i scaled by the cost-weighted factor of the ranges it overlaps
    const int64_t* cost = P.h_chunk_cost.data();
    for (int32_t i = 0; i < n_slices; ++i) {
      const int64_t a = first[i], b = first[i + 1];
      const long double span = (long double)(cost[b] - cost[a]);
      if (b <= a || span <= 0) continue;
      long double acc = 0;
      for (int32_t r = 0; r < world_size; ++r) {
        const int64_t lo = std::max(a, cb[r]), hi = std::min(b, cb[r + 1]);
        if (hi > lo) acc += f[r] * (long double)(cost[hi] - cost[lo]);
      }
      h_ms[i] = (double)(h_ms[i] * acc / span);
    }
  });
}

tc_status tc_partition_measured(const tc_graph* g, int32_t world_size, int32_t n_slices,
                                const double* h_ms, int64_t* h_bounds) {
  return guarded([&] {
    require(g && h_bounds && h_ms, "NULL argument");
    const tc::Plan& P = tc::host_plan(g);
    const tc_status st = tc_partition_chunks(P.h_chunk_seg.data(), P.h_chunk_cost.data(), P.n_chunks,
                                             P.n_long_chunks, n_slices, h_ms, world_size, h_bounds);
    if (st != TC_OK) tc::fail(st, t_last_error);
  });
}

tc_status tc_partition(const tc_graph* g, int32_t world_size, int64_t* h_bounds) {
  return guarded([&] {
    require(g && h_bounds, "NULL argument");
    require(world_size >= 1, "world_size < 1");
    if (world_size == 1) {  // one rank: the whole range (no host chunk arrays needed)
      h_bounds[0] = 0;
      h_bounds[1] = g->plan.S;
      return;
    }
    const tc::Plan& P = tc::host_plan(g);
    // the built-in profile: the classes as two slices (one if a class is empty)
    const int64_t nc = P.n_chunks, nL = P.n_long_chunks;
    const double cl = (double)P.h_chunk_cost[nL], cs = (double)(P.h_chunk_cost[nc] - P.h_chunk_cost[nL]);
    double ms[2];
    int32_t k = 0;
    if (nL > 0) ms[k++] = cl;
    if (nc > nL) ms[k++] = TC_PARTITION_SHORT_RATIO * cs;
    if (k == 0) ms[k++] = 0;
    const tc_status st = tc_partition_chunks(P.h_chunk_seg.data(), P.h_chunk_cost.data(), nc, nL, k,
                                             ms, world_size, h_bounds);
    if (st != TC_OK) tc::fail(st, t_last_error);
  });
}

tc_status tc_plan_chunks(const tc_graph* g, int64_t* h_seg, int64_t* h_cost) {
  return guarded([&] {
    require(g != nullptr, "graph is NULL");
    const tc::Plan& P = tc::host_plan(g);
    if (h_seg) std::copy(P.h_chunk_seg.begin(), P.h_chunk_seg.end(), h_seg);
    if (h_cost) std::copy(P.h_chunk_cost.begin(), P.h_chunk_cost.end(), h_cost);
  });
}

tc_status tc_calibrate(const tc_graph* g, void* stream, int32_t n_slices, double* h_ms) {
  return guarded([&] {
    require(g && h_ms, "NULL argument");
    require(n_slices >= 1, "n_slices < 1");
    const tc::Plan& P = tc::host_plan(g);
    cudaStream_t s = (cudaStream_t)stream;
    for (int32_t i = 0; i < n_slices; ++i) h_ms[i] = 0;
    if (P.n_chunks == 0) return;
    std::vector<int64_t> first(n_slices + 1);
    slice_bounds(P.h_chunk_cost.data(), P.n_chunks, P.n_long_chunks, n_slices, first.data());
    tc::DevBuf<unsigned long long> d(1, s);
    std::vector<cudaEvent_t> ev(n_slices + 1, nullptr);
    struct Guard {
      std::vector<cudaEvent_t>& e;
      ~Guard() {
        for (auto x : e)
          if (x) cudaEventDestroy(x);
      }
    } guard{ev};
    for (auto& e : ev) TC_CUDA(cudaEventCreate(&e));
    tc::count_chunks(g, 0, P.n_chunks, 0, P.S, s, d.get());  // warm-up
    TC_CUDA(cudaEventRecord(ev[0], s));
    for (int32_t i = 0; i < n_slices; ++i) {
      const int64_t c0 = first[i], c1 = first[i + 1];
      if (c1 > c0) tc::count_chunks(g, c0, c1, P.h_chunk_seg[c0], P.h_chunk_seg[c1], s, d.get());
      TC_CUDA(cudaEventRecord(ev[i + 1], s));
    }
    TC_CUDA(cudaEventSynchronize(ev[n_slices]));
    for (int32_t i = 0; i < n_slices; ++i) {
      float ms = 0;
      TC_CUDA(cudaEventElapsedTime(&ms, ev[i], ev[i + 1]));
      h_ms[i] = first[i + 1] > first[i] ? (double)ms : 0.0;
    }
  });
}

// ---------------------------------------------------------------- f2 sharded build
int32_t tc_key_bits(int64_t n) { return tc::key_bits(n < 0 ? 0 : n); }

tc_status tc_shard_canon(const int32_t* d_src, const int32_t* d_dst, int64_t num_edges,
                         int64_t num_vertices, void* stream, uint64_t* d_keys, int64_t* h_count) {
  return guarded([&] {
    require(h_count != nullptr, "h_count is NULL");
    require(num_edges >= 0, "num_edges < 0");
    require(num_edges == 0 || (d_src && d_dst && d_keys), "NULL device pointer");
    require(num_vertices >= 0 && num_vertices <= 0x7fffffffLL,
            "num_vertices must be in [0, 2^31-1] for a sharded build");
    cudaStream_t s = (cudaStream_t)stream;
    tc::reserve_pool((size_t)num_edges * 16, s);
    *h_count = tc::shard_canon(d_src, d_dst, num_edges, num_vertices, s, d_keys);
  });
}

tc_status tc_shard_histogram(const uint64_t* d_keys, int64_t count, int64_t n, int32_t hist_bits,
                             void* stream, int64_t* d_hist) {
  return guarded([&] {
    require(count >= 0 && n >= 0, "count/n < 0");
    require(d_hist && (count == 0 || d_keys), "NULL device pointer");
    require(hist_bits >= 1 && hist_bits <= 24 && hist_bits <= 2 * tc::key_bits(n),
            "hist_bits must be in [1, min(24, 2*tc_key_bits(n))]");
    tc::shard_histogram(d_keys, count, n, hist_bits, (cudaStream_t)stream, d_hist);
  });
}

tc_status tc_shard_cuts(const int64_t* h_hist, int64_t n_buckets, int32_t world_size,
                        int64_t* h_cuts) {
  return guarded([&] {
    require(h_hist && h_cuts, "NULL argument");
    require(n_buckets >= 1, "n_buckets < 1");
    require(world_size >= 1, "world_size < 1");
    std::vector<int64_t> prefix(n_buckets + 1, 0);
    for (int64_t b = 0; b < n_buckets; ++b) {
      require(h_hist[b] >= 0, "negative bucket count");
      prefix[b + 1] = prefix[b] + h_hist[b];
    }
    tc_status st = tc_partition_prefix(prefix.data(), n_buckets, world_size, h_cuts);
    if (st != TC_OK) tc::fail(st, t_last_error);
  });
}

tc_status tc_shard_bounds(const uint64_t* d_keys, int64_t count, int64_t n, int32_t hist_bits,
                          const int64_t* h_cuts, int32_t world_size, void* stream,
                          int64_t* h_bounds) {
  return guarded([&] {
    require(h_cuts && h_bounds && (count == 0 || d_keys), "NULL argument");
    require(count >= 0 && n >= 0, "count/n < 0");
    require(world_size >= 1, "world_size < 1");
    require(hist_bits >= 1 && hist_bits <= 24 && hist_bits <= 2 * tc::key_bits(n),
            "hist_bits must be in [1, min(24, 2*tc_key_bits(n))]");
    for (int32_t r = 0; r < world_size; ++r)
      require(h_cuts[r] <= h_cuts[r + 1], "cuts must be non-decreasing");
    tc::shard_bounds(d_keys, count, n, hist_bits, h_cuts, world_size, (cudaStream_t)stream,
                     h_bounds);
  });
}

tc_status tc_shard_unique(uint64_t* d_keys, int64_t count, int64_t n, void* stream,
                          int64_t* h_count, int32_t* d_degree) {
  return guarded([&] {
    require(h_count != nullptr, "h_count is NULL");
    require(count >= 0 && n >= 0, "count/n < 0");
    require(count == 0 || (d_keys && d_degree), "NULL device pointer");
    *h_count = tc::shard_unique(d_keys, count, n, (cudaStream_t)stream, d_degree);
  });
}

tc_status tc_shard_degree(const uint64_t* d_keys, int64_t count, int64_t n, void* stream,
                          int32_t* d_degree) {
  return guarded([&] {
    require(count >= 0 && n >= 0, "count/n < 0");
    require(count == 0 || (d_keys && d_degree), "NULL device pointer");
    tc::shard_degree(d_keys, count, n, (cudaStream_t)stream, d_degree);
  });
}

tc_status tc_rank_vertices(const int32_t* d_degree, int64_t n, uint32_t flags, void* stream,
                           int32_t* d_rank, int32_t* d_perm, int64_t* h_n_active) {
  return guarded([&] {
    require(h_n_active != nullptr, "h_n_active is NULL");
    require(n >= 0 && n <= 0x7fffffffLL, "n must be in [0, 2^31-1]");
    require(n == 0 || (d_degree && d_rank && d_perm), "NULL device pointer");
    require((flags & ~TC_KEEP_ISOLATED) == 0, "unknown flag bits");
    *h_n_active = tc::shard_rank(d_degree, n, flags, (cudaStream_t)stream, d_rank, d_perm);
  });
}

tc_status tc_shard_orient(const uint64_t* d_keys, int64_t count, int64_t n, const int32_t* d_rank,
                          int64_t n_active, void* stream, uint64_t* d_okeys) {
  return guarded([&] {
    require(count >= 0 && n >= 0 && n_active >= 0 && n_active <= n, "bad sizes");
    require(count == 0 || (d_keys && d_rank && d_okeys), "NULL device pointer");
    require(count == 0 || d_keys != d_okeys, "d_okeys may not alias d_keys");
    tc::shard_orient(d_keys, count, n, d_rank, n_active, (cudaStream_t)stream, d_okeys);
  });
}

tc_status tc_sort_keys(uint64_t* d_keys, int64_t count, int64_t n, void* stream) {
  return guarded([&] {
    require(count >= 0 && n >= 0, "count/n < 0");
    require(count == 0 || d_keys, "NULL device pointer");
    tc::sort_keys(d_keys, count, n, (cudaStream_t)stream);
  });
}

tc_status tc_build_from_oriented(const uint64_t* d_okeys, int64_t m, const int32_t* d_perm,
                                 int64_t n_active, int64_t n_input, const tc_options* opts,
                                 void* stream, tc_graph** out) {
  if (out) *out = nullptr;
  tc_graph* g = nullptr;
  tc_status st = guarded([&] {
    require(out != nullptr, "out is NULL");
    require(m >= 0 && n_active >= 0 && n_input >= n_active && n_input <= 0x7fffffffLL, "bad sizes");
    require(m == 0 || d_okeys, "d_okeys is NULL");
    require(n_active == 0 || d_perm, "d_perm is NULL");
    const tc::Options opt = tc::resolve_options(opts);
    cudaStream_t s = (cudaStream_t)stream;
    tc::reserve_pool((size_t)m * 40, s);
    g = new tc_graph();
    tc::build_from_oriented(d_okeys, m, d_perm, n_active, n_input, opt, s, g);
  });
  if (st != TC_OK) {
    if (g) {
      cudaStreamSynchronize((cudaStream_t)stream);
      delete g;
    }
    return st;
  }
  *out = g;
  return TC_OK;
}

void tc_free(tc_graph* g) {
  if (!g) return;
  // the graph's own build and replans completed before they returned; wait
  // for the work other streams enqueued on it, then free stream-ordered
  {
    std::lock_guard<std::mutex> lk(g->use_mu);
    for (auto& u : g->uses) {
      cudaEventSynchronize(u.ev);
      cudaEventDestroy(u.ev);
    }
    g->uses.clear();
  }
  rebind(g, nullptr);
  delete g;
}

tc_status tc_counters(uint64_t* h_counters, int32_t reset) {
  return guarded([&] {
    require(h_counters != nullptr, "NULL argument");
    tc::read_counters(h_counters, reset != 0);
  });
}

tc_status tc_release_memory(void) {
  return guarded([&] { tc::trim_pools(); });
}

const char* tc_last_error(void) { return t_last_error.c_str(); }

const char* tc_version(void) { return "b200tc 0.1 sm_100a"; }

}  // extern "C"

// tc_internal.cuh — shared internals of libtc.so (not part of the C-ABI).
//
// Product path only: nothing here is shared with oracle/ (DESIGN.md §3).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <utility>
#include <vector>

#include "tc.h"

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
void* dev_alloc(size_t bytes, cudaStream_t s);  // throws TC_ERR_OUT_OF_MEMORY
void dev_free(void* p, size_t bytes, cudaStream_t s);

// Owning device buffer (stream-ordered free on the stream it was made on).
template <class T>
struct DevBuf {
  T* p = nullptr;
  size_t n = 0;
  cudaStream_t s = nullptr;
  DevBuf() = default;
  DevBuf(size_t count, cudaStream_t st) : n(count), s(st) {
    if (count) p = static_cast<T*>(dev_alloc(count * sizeof(T), st));
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

// ---------------------------------------------------------------- options
struct Options {
  int chunk_cost = 16384;
  int seg_cost = 4;
  int huge_degree = 8192;
  int block_threads = 512;
  int hash_shift = 1;
};
Options resolve_options(const tc_options* o);

// ---------------------------------------------------------------- plan
// The dispatch plan.  Units:
//   segment s  = one LIVE oriented edge (u,v) (suffix of N+(u) after v is
//                non-empty and d+(v) > 0), in (v, position) order; its keys
//                are col[p+1 .. row_end(u)), the suffix of P:359.
//   group g    = one distinct head vertex v over the segments; its table is
//                N+(v) = col[row_ptr[v] .. row_ptr[v+1]).
//   flat key k = global index over all segments' keys, k in
//                [key_prefix[s], key_prefix[s+1]) belongs to s and lives at
//                col[seg_base[s] + k].
//   chunk c    = segments [chunk_seg[c], chunk_seg[c+1]) of near-equal cost.
struct PlanView {
  const int32_t* col;
  const int64_t* key_prefix;   // [S+1]
  const int64_t* seg_base;     // [S]  = (p+1) - key_prefix[s]
  const int32_t* seg_group;    // [S]
  const int64_t* ins_prefix;   // [G+1] prefix of d+(v)
  const int64_t* grp_ibase;    // [G]  = row_ptr[v] - ins_prefix[g]
  const int64_t* slot_prefix;  // [G+1] prefix of hash slots (0 for huge groups)
  const int32_t* grp_tmax;     // [G]  max element of N+(v)
  const int64_t* chunk_seg;    // [C+1]
};

struct Plan {
  Options opt;
  int64_t S = 0, G = 0, n_chunks = 0, keys_total = 0;
  DevBuf<int64_t> key_prefix, seg_base, ins_prefix, grp_ibase, slot_prefix, chunk_seg;
  DevBuf<int32_t> seg_group, grp_tmax;
  std::vector<int64_t> h_chunk_seg;
  int64_t smem_bytes = 0;
  int grid = 0, block = 0;
};

}  // namespace tc

struct tc_graph {
  int64_t n_input = 0, n = 0, m = 0, max_out = 0;
  int bits = 1;  // bits of a vertex id in [0, n)
  tc::DevBuf<int64_t> row_ptr;
  tc::DevBuf<int32_t> col, perm;
  tc::Plan plan;
  uint64_t b_itc = 0;
  float ms[6] = {0, 0, 0, 0, 0, 0};
};

namespace tc {

// tc_build.cu
void build_graph(const int32_t* d_src, const int32_t* d_dst, int64_t m_gen, int64_t n,
                 uint32_t flags, const Options& opt, cudaStream_t s, tc_graph* g);
void build_plan(tc_graph* g, const Options& opt, cudaStream_t s);

// tc_count.cu
void count_chunks(const tc_graph* g, int64_t c_begin, int64_t c_end, int64_t e_begin,
                  int64_t e_end, cudaStream_t s, unsigned long long* d_out);
int count_occupancy(int block, int64_t smem_bytes);  // CTAs per SM (0 = cannot launch)
int max_smem_per_block();
int num_sms();

}  // namespace tc

// tc_build.cu — preprocessing: SURVEY.md §8(a) rows a1..a6 on the GPU.
//
//   a1 validate + canonicalise + drop self-loops
//   a2 radix sort + unique                          ("resolving duplicate edges")
//   a3 undirected degree                            (P:108 degree ordering)
//   a4 rank by (degree, id), relabel, drop isolated ("u < v")
//   a5 orient u -> v iff rank u < rank v, CSR
//   a6 dispatch plan (live edges grouped by head v, hash sizes, cost chunks)
//
// Every pass is a streaming integer pass (HBM bound); the sorts are CUB's
// onesweep radix sort on the minimal bit width (2*ceil(log2 n) bits).  The
// only host round trips are the counts that size the next allocation.
#include <cub/cub.cuh>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <string>

#include "tc_internal.cuh"

namespace tc {
namespace {

constexpr int TPB = 256;

unsigned grid_for(int64_t n) {
  int64_t b = (n + TPB - 1) / TPB;
  return (unsigned)std::max<int64_t>(1, std::min<int64_t>(b, 148 * 32));
}

int bits_for(int64_t n) {  // bits so that every id in [0, n) fits
  int b = 1;
  while ((int64_t(1) << b) < n) ++b;
  return b;
}

template <class F>
void cub_run(cudaStream_t s, F f) {
  size_t bytes = 0;
  TC_CUDA(f(nullptr, bytes));
  DevBuf<char> tmp(bytes ? bytes : 16, s);
  TC_CUDA(f(tmp.get(), bytes));
}

// TC_VERBOSE=1: plan sub-phase trace on stderr (host clock after a stream sync).
struct Trace {
  bool on;
  cudaStream_t s;
  std::chrono::steady_clock::time_point t0;
  explicit Trace(cudaStream_t st) : on(std::getenv("TC_VERBOSE") != nullptr), s(st) {
    if (on) {
      cudaStreamSynchronize(s);
      t0 = std::chrono::steady_clock::now();
    }
  }
  void operator()(const char* what) {
    if (!on) return;
    cudaStreamSynchronize(s);
    auto t = std::chrono::steady_clock::now();
    fprintf(stderr, "[tc] %-28s %8.2f ms\n", what,
            std::chrono::duration<double, std::milli>(t - t0).count());
    t0 = t;
  }
};

// The build's 64-bit key sorts (a2, a5, the host entry's pieces, the sharded
// build) run CUB's onesweep with 256 threads x 22 keys per thread instead of
// its sm_100 default (384 x 15): 268 M keys on 48 bits in 11.6 vs 16.3 ms
// (scripts/sort_bench.cu, profiles/r4d_sort_bench.txt).  TC_SORT=cub keeps the
// default policy.  (A hand-written reduce-then-scan LSD sort with
// __match_any_sync ranking measured 25.5 ms, the key/value form 37.6 vs 9.1.)
using SortOffset = unsigned long long;
struct KeySortHub {
  using Base = cub::detail::radix::policy_hub<uint64_t, cub::NullType, SortOffset>::Policy1000;
  struct P : cub::ChainedPolicy<1000, P, P> {
    static constexpr bool ONESWEEP = true;
    static constexpr int ONESWEEP_RADIX_BITS = 8;
    using HistogramPolicy = Base::HistogramPolicy;
    using ExclusiveSumPolicy = Base::ExclusiveSumPolicy;
    // nominal items for 4-B keys (CUB scales by the key size: 22 per thread)
    using OnesweepPolicy =
        cub::AgentRadixSortOnesweepPolicy<256, 44, uint64_t, 1, cub::RADIX_RANK_MATCH_EARLY_COUNTS_ANY,
                                          cub::BLOCK_SCAN_RAKING_MEMOIZE, cub::RADIX_SORT_STORE_DIRECT, 8>;
    using ScanPolicy = Base::ScanPolicy;
    using DownsweepPolicy = Base::DownsweepPolicy;
    using AltDownsweepPolicy = Base::AltDownsweepPolicy;
    using UpsweepPolicy = Base::UpsweepPolicy;
    using AltUpsweepPolicy = Base::AltUpsweepPolicy;
    using SingleTilePolicy = Base::SingleTilePolicy;
    using SegmentedPolicy = Base::SegmentedPolicy;
    using AltSegmentedPolicy = Base::AltSegmentedPolicy;
  };
  using MaxPolicy = P;
};

void sort_keys_u64(cub::DoubleBuffer<uint64_t>& db, int64_t n, int end_bit, cudaStream_t s) {
  static const bool cub_default = [] {
    const char* v = std::getenv("TC_SORT");
    return v && std::string(v) == "cub";
  }();
  if (cub_default) {
    cub_run(s, [&](void* t, size_t& b) { return cub::DeviceRadixSort::SortKeys(t, b, db, n, 0, end_bit, s); });
    return;
  }
  cub::DoubleBuffer<cub::NullType> dv;
  cub_run(s, [&](void* t, size_t& b) {
    return cub::DispatchRadixSort<false, uint64_t, cub::NullType, SortOffset, KeySortHub>::Dispatch(
        t, b, db, dv, (SortOffset)n, 0, end_bit, true, s);
  });
}

template <class T>
T d2h(const T* d, cudaStream_t s) {
  T h;
  TC_CUDA(cudaMemcpyAsync(&h, d, sizeof(T), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
  return h;
}

// ------------------------------------------------------------------ a1
// key = (min << bits) | max for a valid non-loop pair, SENT otherwise.
__global__ void k_canon(const int32_t* __restrict__ src, const int32_t* __restrict__ dst,
                        int64_t m, int64_t n, int bits, uint64_t sent,
                        uint64_t* __restrict__ key, int* __restrict__ err) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m;
       i += (int64_t)gridDim.x * blockDim.x) {
    int64_t a = src[i], b = dst[i];
    uint64_t k = sent;
    if (a < 0 || b < 0 || a >= n || b >= n) {
      *err = 1;
    } else if (a != b) {
      uint64_t lo = (uint64_t)min(a, b), hi = (uint64_t)max(a, b);
      k = (lo << bits) | hi;
    }
    key[i] = k;
  }
}

// a1 + a2 by hashing (small inputs, see build_graph): the canonical keys only need
// to be UNIQUE here — a3 (degree) and a5 (orient, then a full sort) do not
// care about their order — so a linear-probing u64 hash set (load <= 1/2)
// replaces the 2*ceil(log2 n)-bit radix sort.  EMPTY = all ones (never a
// valid key: lo < hi).  Exact: a key is inserted iff it is not yet present.
__device__ __forceinline__ uint64_t mix64(uint64_t x) {
  x ^= x >> 31;
  x *= 0x7fb5d329728ea185ull;
  x ^= x >> 27;
  return x;
}

__global__ void k_canon_hash(const int32_t* __restrict__ src, const int32_t* __restrict__ dst,
                             int64_t m, int64_t n, int bits, uint64_t* __restrict__ table,
                             int log2cap, int* __restrict__ err) {
  const uint64_t mask = (uint64_t(1) << log2cap) - 1;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t a = src[i], b = dst[i];
    if (a < 0 || b < 0 || a >= n || b >= n) {
      *err = 1;
      continue;
    }
    if (a == b) continue;
    const uint64_t k = ((uint64_t)min(a, b) << bits) | (uint64_t)max(a, b);
    uint64_t h = mix64(k) >> (64 - log2cap);
    for (;;) {
      const unsigned long long cur = ((volatile unsigned long long*)table)[h];
      if (cur == k) break;
      if (cur == ~0ull) {
        const unsigned long long prev =
            atomicCAS(reinterpret_cast<unsigned long long*>(table + h), ~0ull, (unsigned long long)k);
        if (prev == ~0ull || prev == k) break;
      }
      h = (h + 1) & mask;
    }
  }
}

struct NotEmpty {
  __host__ __device__ bool operator()(const uint64_t& x) const { return x != ~0ull; }
};

// {err, n_selected, last key} for the single host round trip after a2.
struct UniqTail {
  int err;
  int pad;
  int64_t nsel;
  uint64_t last;
};
__global__ void k_uniq_tail(const int* err, const int64_t* nsel, const uint64_t* keys,
                            UniqTail* out) {
  out->err = *err;
  out->nsel = *nsel;
  out->last = *nsel > 0 ? keys[*nsel - 1] : 0;
}

// ------------------------------------------------------------------ a3
// The first endpoints of sorted keys come in runs: lanes holding the same
// one add their count with one atomic (__match_any_sync); the second
// endpoint takes one atomic per key.  Exact for any key order.
__global__ void k_degree(const uint64_t* __restrict__ key, int64_t m, int bits,
                         int32_t* __restrict__ deg) {
  const uint64_t mask = (uint64_t(1) << bits) - 1;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t m_round = (m + 31) & ~int64_t(31);  // whole warps stay converged
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m_round; i += stride) {
    const bool in = i < m;
    const uint64_t k = in ? key[i] : ~0ull;
    const unsigned a = in ? (unsigned)(k >> bits) : 0xffffffffu;
    const unsigned same = __match_any_sync(0xffffffffu, a);
    if (in && (threadIdx.x & 31) == __ffs(same) - 1) atomicAdd(&deg[a], __popc(same));
    if (in) atomicAdd(&deg[k & mask], 1);
  }
}

// ------------------------------------------------------------------ a4
// vertex key = (deg << bits) | v; isolated vertices get SENTV (sorted last)
// unless TC_KEEP_ISOLATED.  Counts the kept vertices into *n_act.
__global__ void k_vkey(const int32_t* __restrict__ deg, int64_t n, int bits, int keep,
                       uint64_t sentv, uint64_t* __restrict__ vkey,
                       unsigned long long* __restrict__ n_act) {
  for (int64_t base = blockIdx.x * (int64_t)blockDim.x; base < n;
       base += (int64_t)gridDim.x * blockDim.x) {
    int64_t v = base + threadIdx.x;
    int act = 0;
    if (v < n) {
      int64_t d = deg[v];
      act = keep || d > 0;
      vkey[v] = act ? (((uint64_t)d << bits) | (uint64_t)v) : sentv;
    }
    int c = __syncthreads_count(act);
    if (threadIdx.x == 0 && c) atomicAdd(n_act, (unsigned long long)c);
  }
}

__global__ void k_perm(const uint64_t* __restrict__ vkey, int64_t n_act, int bits,
                       int32_t* __restrict__ perm, int32_t* __restrict__ rank) {
  const uint64_t mask = (uint64_t(1) << bits) - 1;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n_act;
       i += (int64_t)gridDim.x * blockDim.x) {
    int32_t v = (int32_t)(vkey[i] & mask);
    perm[i] = v;
    rank[v] = (int32_t)i;
  }
}

// ------------------------------------------------------------------ a5
__global__ void k_orient(const uint64_t* __restrict__ key, int64_t m, int bits,
                         const int32_t* __restrict__ rank, int bits2,
                         uint64_t* __restrict__ okey) {
  const uint64_t mask = (uint64_t(1) << bits) - 1;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m;
       i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t k = key[i];
    uint64_t ra = (uint64_t)rank[k >> bits], rb = (uint64_t)rank[k & mask];
    okey[i] = ra < rb ? ((ra << bits2) | rb) : ((rb << bits2) | ra);
  }
}

// CSR of sorted oriented keys; also the row of every position (rowid, the
// plan's first input: one write here instead of a separate pass over rows).
__global__ void k_csr(const uint64_t* __restrict__ okey, int64_t m, int64_t n, int bits2,
                      int32_t* __restrict__ col, int64_t* __restrict__ row_ptr,
                      int32_t* __restrict__ rowid) {
  const uint64_t mask = (uint64_t(1) << bits2) - 1;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m;
       i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t k = okey[i];
    int64_t u = (int64_t)(k >> bits2);
    col[i] = (int32_t)(k & mask);
    rowid[i] = (int32_t)u;
    int64_t prev = i ? (int64_t)(okey[i - 1] >> bits2) : -1;
    for (int64_t x = prev + 1; x <= u; ++x) row_ptr[x] = i;
    if (i == m - 1)
      for (int64_t x = u + 1; x <= n; ++x) row_ptr[x] = m;
  }
}


__global__ void k_fill_i64(int64_t* p, int64_t n, int64_t v) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    p[i] = v;
}

__global__ void k_max_outdeg(const int64_t* __restrict__ row_ptr, int64_t n,
                             unsigned long long* out) {
  typedef cub::BlockReduce<unsigned long long, TPB> BR;
  __shared__ typename BR::TempStorage tmp;
  unsigned long long mx = 0;
  for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n;
       u += (int64_t)gridDim.x * blockDim.x)
    mx = max(mx, (unsigned long long)(row_ptr[u + 1] - row_ptr[u]));
  unsigned long long r = BR(tmp).Reduce(mx, cub::Max());
  if (threadIdx.x == 0) atomicMax(out, r);
}

// ------------------------------------------------------------------ a6
__global__ void k_rowid(const int64_t* __restrict__ row_ptr, int64_t n,
                        int32_t* __restrict__ rowid) {
  for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n;
       u += (int64_t)gridDim.x * blockDim.x)
    for (int64_t p = row_ptr[u], e = row_ptr[u + 1]; p < e; ++p) rowid[p] = (int32_t)u;
}

// Per row v: {min N+(v), max N+(v), d+(v), 0} (rows are sorted), {INT_MAX,
// -1, 0, 0} if empty: the one 16-B record k_edge_trim reads at random per edge
// (instead of row_ptr[v], row_ptr[v+1] and the two ends in col).
__global__ void k_vmm(const int64_t* __restrict__ row_ptr, const int32_t* __restrict__ col,
                      int64_t n, int4* __restrict__ vmm) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t a = row_ptr[v], b = row_ptr[v + 1];
    vmm[v] = b > a ? make_int4(col[a], col[b - 1], (int)(b - a), 0) : make_int4(0x7fffffff, -1, 0, 0);
  }
}

__device__ __forceinline__ int64_t lower_bound_i32(const int32_t* __restrict__ a, int64_t lo,
                                                   int64_t hi, int32_t x) {
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (a[mid] < x) lo = mid + 1; else hi = mid;
  }
  return lo;
}

__device__ __forceinline__ int64_t upper_bound_i32(const int32_t* __restrict__ a, int64_t lo,
                                                   int64_t hi, int32_t x) {
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (a[mid] <= x) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// Per oriented edge p = (u, v): the keys are the suffix of N+(u) after v,
// col[p+1, row_end(u)), trimmed to [min N+(v), max N+(v)] because a
// key outside that range cannot be in N+(v) (both lists sorted; exact, C-12).
// Live iff the trimmed suffix is non-empty.  Emits the plan's sort key
// (class above head v; dead edges get `dead`, which sorts last) and the
// packed value (trimmed start << 24 | length).  stats: [0] B_ITC edge part
// (untrimmed), [1] trimmed keys, [2] live, [3] live long,
// [4] trimmed keys of the long class.
__global__ void k_edge_trim(const int64_t* __restrict__ row_ptr, const int32_t* __restrict__ col,
                            const int32_t* __restrict__ rowid, const int4* __restrict__ vmm,
                            int64_t m, int long_min, int bits,
                            uint32_t dead, uint32_t* __restrict__ skey, uint64_t* __restrict__ sval,
                            unsigned long long* stats, int hash_dmax, int bitmap_factor) {
  typedef cub::BlockReduce<unsigned long long, TPB> BR;
  __shared__ typename BR::TempStorage tmp;
  unsigned long long b = 0, keys = 0, nl = 0, nlong = 0, klong = 0;
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < m;
       p += (int64_t)gridDim.x * blockDim.x) {
    const int32_t u = rowid[p], v = col[p];
    const int64_t rend = row_ptr[u + 1], suf = rend - p - 1;
    const int4 w = vmm[v];  // {min N+(v), max N+(v), d+(v)}
    b += 4ull * (unsigned long long)(suf + w.z) + 12ull;
    int64_t lo = p + 1, len = 0;
    if (suf > 0 && w.z > 0) {
      lo = lower_bound_i32(col, p + 1, rend, w.x);
      len = upper_bound_i32(col, lo, rend, w.y) - lo;
    }
    // long class: len >= long_min; with TC_LONG_HASH_DMAX = D > 0, an edge
    // whose head gets a hash table (no bitmap) with d+(v) <= D is flattened
    // with the short class instead (tiny tables, few edges per group: the
    // producer-bound head of the long class)
    bool lng = len >= long_min;
    if (hash_dmax > 0 && lng && w.z <= hash_dmax)
      lng = (w.x >> 5) < (1 << 25) &&
            (int64_t)((w.y >> 5) - (w.x >> 5) + 1) <= (int64_t)bitmap_factor * w.z;
    const uint32_t cls = lng ? 0u : 1u;
    skey[p] = len > 0 ? ((cls << bits) | (uint32_t)v) : dead;
    sval[p] = ((uint64_t)lo << 24) | (uint64_t)len;  // len <= d+(u) < 2^24
    keys += (unsigned long long)len;
    nl += len > 0;
    nlong += lng;
    klong += lng ? (unsigned long long)len : 0ull;
  }
  unsigned long long r0 = BR(tmp).Sum(b);
  __syncthreads();
  unsigned long long r1 = BR(tmp).Sum(keys);
  __syncthreads();
  unsigned long long r2 = BR(tmp).Sum(nl);
  __syncthreads();
  unsigned long long r3 = BR(tmp).Sum(nlong);
  __syncthreads();
  unsigned long long r4 = BR(tmp).Sum(klong);
  if (threadIdx.x == 0) {
    atomicAdd(&stats[0], r0);
    atomicAdd(&stats[1], r1);
    atomicAdd(&stats[2], r2);
    atomicAdd(&stats[3], r3);
    atomicAdd(&stats[4], r4);
  }
}

// 1 at the first segment of each group (its sort key differs from the
// previous one): read on the fly by the group-index scan (no mark array).
struct GroupStart {
  const uint32_t* key;
  __host__ __device__ int32_t operator()(int64_t s) const {
    return (s == 0 || key[s] != key[s - 1]) ? 1 : 0;
  }
};

// Per segment (sorted live edge): start, length, group, work units; per
// group (at its first segment): row start, d+(v) and its table.
__global__ void k_seg_fill(const uint32_t* __restrict__ key, const uint64_t* __restrict__ val,
                           const int32_t* __restrict__ gincl, int64_t S, int64_t S_long,
                           int bits, const int64_t* __restrict__ row_ptr,
                           int huge_degree, int table_factor, int bitmap_factor,
                           int64_t max_slots_long, int64_t max_slots_short,
                           const int32_t* __restrict__ col,
                           int32_t* __restrict__ grp_code, uint32_t* __restrict__ seg_start,
                           int32_t* __restrict__ seg_len, int32_t* __restrict__ seg_group,
                           uint32_t* __restrict__ units, int64_t* __restrict__ grp_row,
                           int64_t* __restrict__ grp_d, int64_t* __restrict__ grp_slots,
                           int seg_cost, int64_t* __restrict__ cost,
                           unsigned long long* __restrict__ units_total) {
  typedef cub::BlockReduce<unsigned long long, TPB> BR;
  __shared__ typename BR::TempStorage tmp;
  const uint32_t mask = (uint32_t)((1ull << bits) - 1);
  unsigned long long usum = 0;
  for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < S;
       s += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t x = val[s];
    const int32_t g = gincl[s] - 1;
    const int32_t len = (int32_t)(x & 0xFFFFFFu);
    seg_group[s] = g;
    seg_start[s] = (uint32_t)(x >> 24);  // < m < 2^32
    seg_len[s] = len;
    const uint32_t u = s < S_long ? (uint32_t)((len + 31) & ~31) : (uint32_t)len;
    units[s] = u;
    usum += u;
    // the segment's plan cost (k_chunk_bounds): seg_cost + its units, plus
    // its group's d+(v) and table words at the group's first segment
    int64_t c = seg_cost + (int64_t)u;
    if (s == 0 || key[s] != key[s - 1]) {
      const int64_t v = key[s] & mask;
      const int64_t rs = row_ptr[v], d = row_ptr[v + 1] - rs;
      grp_row[g] = rs;
      grp_d[g] = d;
      // Table of N+(v), in 32-bit words (0 = huge: probed in global memory):
      //  bitmap: one bit per rank of the window [min N+(v), max N+(v)] at word
      //    granularity, when that is at most bitmap_factor * d words (one
      //    probe per key); code = -(first word);
      //  hash: table_factor * d slots (load <= 1/table_factor, > d so a
      //    linear probe always meets an empty slot); code = slots.
      // Sizes are multiples of 4 for 16-B initialisation.
      // The cap is the SMEM of the class's own kernel (a long group's table
      // lives in a k_count slot, a short group's in a k_count_flat chunk); a
      // hash table that would exceed it at table_factor falls back to load
      // 1/3, then 1/2, before the group is declared huge (C4's hubs, d+ up to
      // 4,218: with one cap for both classes they went to global binary search).
      const int64_t maxs = s < S_long ? max_slots_long : max_slots_short;
      int64_t slots = 0;
      int32_t code = 0;
      if (d <= huge_degree) {
        const int64_t w0 = col[rs] >> 5, w1 = col[rs + d - 1] >> 5;
        const int64_t bw = (w1 - w0 + 1 + 3) & ~int64_t(3);
        // (the first word must fit the count kernel's 26-bit tile code)
        if (bitmap_factor > 0 && w0 < (1 << 25) && w1 - w0 + 1 <= (int64_t)bitmap_factor * d &&
            bw <= maxs) {
          slots = bw;
          code = -(int32_t)w0;
        } else {
          int64_t want = d * table_factor;
          if (want > maxs) want = 3 * d;  // load 1/3: two-choice inserts still rarely fail
          if (want > maxs) want = 2 * d;
          if (want < d + 1) want = d + 1;
          slots = (want + 3) & ~int64_t(3);
          code = (int32_t)slots;
          if (slots > maxs) slots = code = 0;
        }
      }
      grp_code[g] = code;
      grp_slots[g] = slots;
      c += d + slots;
    }
    cost[s] = c;
  }
  const unsigned long long r = BR(tmp).Sum(usum);
  if (threadIdx.x == 0) atomicAdd(units_total, r);
}


__global__ void k_grp_ibase(const int64_t* __restrict__ grp_row,
                            const int64_t* __restrict__ ins_prefix, int64_t G,
                            int64_t* __restrict__ ibase) {
  for (int64_t g = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; g < G;
       g += (int64_t)gridDim.x * blockDim.x)
    ibase[g] = grp_row[g] - ins_prefix[g];
}

// Chunks never straddle the class boundary S_long: long chunk c < nL starts
// at the first segment whose cost prefix reaches c*CL; short chunk nL + j at
// the first segment of [S_long, S) whose prefix reaches prefix[S_long] + j*CS.
__global__ void k_chunk_bounds(const int64_t* __restrict__ cost_prefix, int64_t S_long,
                               int64_t S, int64_t nL, int64_t nS, int64_t CL, int64_t CS,
                               int64_t* __restrict__ chunk_seg) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c <= nL + nS;
       c += (int64_t)gridDim.x * blockDim.x) {
    if (c == nL + nS) {
      chunk_seg[c] = S;
      continue;
    }
    int64_t lo, hi, target;
    if (c < nL) {
      lo = 0;
      hi = S_long;
      target = c * CL;
    } else {
      lo = S_long;
      hi = S;
      target = cost_prefix[S_long] + (c - nL) * CS;
    }
    while (lo < hi) {  // first s with prefix[s] >= target
      int64_t mid = (lo + hi) >> 1;
      if (cost_prefix[mid] < target) lo = mid + 1; else hi = mid;
    }
    chunk_seg[c] = lo;
  }
}

// SMEM-capped split of the cost chunks (one thread per chunk, sequential
// over its edges): a piece grows edge by edge while its slot layout
// (chunk_smem_bytes: edges, groups, hash slots, long-class tiles) fits
// `limit`.  Pass 1 (bounds == nullptr) counts pieces per chunk and the
// largest piece; pass 2 writes each piece's first edge at off[c] + j.
__global__ void k_split(const int64_t* __restrict__ chunk_seg, int64_t n_chunks, int64_t nL,
                        const int32_t* __restrict__ seg_group,
                        const int64_t* __restrict__ slot_prefix,
                        const uint32_t* __restrict__ key_prefix, int64_t limit_long,
                        int64_t limit_short, int64_t* __restrict__ pieces,
                        const int64_t* __restrict__ off, int64_t* __restrict__ bounds,
                        unsigned long long* need_max) {  // need_max[0] long, [1] short
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n_chunks;
       c += (int64_t)gridDim.x * blockDim.x) {
    const int64_t sa = chunk_seg[c], sb = chunk_seg[c + 1];
    int64_t o = bounds ? off[c] : 0, cnt = 0;
    if (sa >= sb) {  // an empty chunk stays one (empty) piece
      if (bounds) bounds[o] = sa;
      else pieces[c] = 1;
      continue;
    }
    const bool is_long = c < nL;
    const int64_t limit = is_long ? limit_long : limit_short;
    unsigned long long* nm = need_max ? need_max + (is_long ? 0 : 1) : nullptr;
    {
      // fast path: the whole chunk fits one slot (all but the outliers) —
      // its layout follows from the prefixes in O(1), no walk over its edges
      const int64_t ga = seg_group[sa], gb = seg_group[sb - 1];
      // key_prefix is mod 2^32; a chunk's units are < 2^32
      const int64_t tiles = is_long ? (int64_t)((key_prefix[sb] - key_prefix[sa]) >> 5) : 0;
      const int64_t need = chunk_smem_bytes(sb - sa, gb - ga + 1, slot_prefix[gb + 1] - slot_prefix[ga], tiles);
      if (need <= limit) {
        if (bounds) bounds[o] = sa;
        else {
          atomicMax(nm, (unsigned long long)need);
          pieces[c] = 1;
        }
        continue;
      }
    }
    // outlier: cut it into pieces, each the longest run [p0, e) whose layout
    // fits `limit` (at least one edge).  The layout size grows with e, so e is
    // binary-searched (the pieces a walk edge by edge would cut).
    auto need_of = [&](int64_t a, int64_t e) {
      const int64_t g0 = seg_group[a], g1 = seg_group[e - 1];
      const int64_t tiles = is_long ? (int64_t)((key_prefix[e] - key_prefix[a]) >> 5) : 0;
      return chunk_smem_bytes(e - a, g1 - g0 + 1, slot_prefix[g1 + 1] - slot_prefix[g0], tiles);
    };
    int64_t p0 = sa;
    for (;;) {
      int64_t lo = p0 + 1, hi = sb;
      if (need_of(p0, lo) <= limit) {
        while (lo < hi) {  // largest e in [p0 + 1, sb] with need <= limit
          const int64_t mid = (lo + hi + 1) >> 1;
          if (need_of(p0, mid) <= limit) lo = mid; else hi = mid - 1;
        }
      }
      if (lo >= sb) break;  // [p0, sb) is the last piece
      if (bounds) bounds[o + cnt] = p0;
      else atomicMax(nm, (unsigned long long)need_of(p0, lo));
      ++cnt;
      p0 = lo;
    }
    const int64_t ok_need = need_of(p0, sb);
    if (bounds) bounds[o + cnt] = p0;
    else {
      atomicMax(nm, (unsigned long long)ok_need);
      pieces[c] = cnt + 1;
    }
  }
}

// Per chunk: the plan cost prefix at its first edge (the host copy drives
// tc_partition's cost split), and the table rows / group visits its producers
// read (the method's own bytes).  stats: [0] sum of d+(v)
// over (chunk, group) pairs, [1] number of such pairs.
__global__ void k_chunk_meta(const int64_t* __restrict__ chunk_seg, int64_t nc, int64_t nL,
                             const int32_t* __restrict__ seg_group,
                             const int64_t* __restrict__ ins_prefix,
                             const int64_t* __restrict__ cost_prefix,
                             int64_t* __restrict__ chunk_cost, unsigned long long* stats) {
  typedef cub::BlockReduce<unsigned long long, TPB> BR;
  __shared__ typename BR::TempStorage tmp;
  unsigned long long tw = 0, gv = 0, twl = 0, gvl = 0;
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c <= nc;
       c += (int64_t)gridDim.x * blockDim.x) {
    const int64_t sa = chunk_seg[c];
    chunk_cost[c] = cost_prefix[sa];
    if (c == nc) continue;
    const int64_t sb = chunk_seg[c + 1];
    if (sa >= sb) continue;
    const int64_t ga = seg_group[sa], gb = seg_group[sb - 1];
    const unsigned long long w = (unsigned long long)(ins_prefix[gb + 1] - ins_prefix[ga]);
    const unsigned long long v = (unsigned long long)(gb - ga + 1);
    tw += w;
    gv += v;
    if (c < nL) {
      twl += w;
      gvl += v;
    }
  }
  unsigned long long r[4] = {tw, gv, twl, gvl};
  for (int i = 0; i < 4; ++i) {
    const unsigned long long x = BR(tmp).Sum(r[i]);
    __syncthreads();
    if (threadIdx.x == 0) atomicAdd(&stats[i], x);
  }
}

// ------------------------------------------------------------------ f2
// Sharded preprocessing: range split of sorted keys.
__device__ __forceinline__ int64_t lower_bound_u64(const uint64_t* __restrict__ a, int64_t n,
                                                   uint64_t x) {
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (a[mid] < x) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// hist[b] = #keys with key >> shift == b, by two binary searches per bucket
// (the keys are sorted: no atomics, deterministic).
__global__ void k_key_hist(const uint64_t* __restrict__ keys, int64_t cnt, int shift, int64_t nb,
                           int64_t* __restrict__ hist) {
  for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < nb;
       b += (int64_t)gridDim.x * blockDim.x) {
    const int64_t lo = lower_bound_u64(keys, cnt, (uint64_t)b << shift);
    const int64_t hi = b + 1 < nb ? lower_bound_u64(keys, cnt, (uint64_t)(b + 1) << shift) : cnt;
    hist[b] = hi - lo;
  }
}

// pos[r] = first key whose bucket >= cut[r] (cut[r] == nb -> cnt).
__global__ void k_key_bounds(const uint64_t* __restrict__ keys, int64_t cnt, int shift, int64_t nb,
                             const int64_t* __restrict__ cut, int np, int64_t* __restrict__ pos) {
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r < np) pos[r] = cut[r] >= nb ? cnt : lower_bound_u64(keys, cnt, (uint64_t)cut[r] << shift);
}

__global__ void k_set_i64(int64_t* p, int64_t v) { *p = v; }

// exclusive prefix of `in` (length n) into out[0..n] (out[0] = 0, out[n] = total)
void exclusive_prefix(const int64_t* in, int64_t n, int64_t* out, cudaStream_t s) {
  TC_CUDA(cudaMemsetAsync(out, 0, sizeof(int64_t), s));
  if (n == 0) return;
  cub_run(s, [&](void* t, size_t& b) {
    return cub::DeviceScan::InclusiveSum(t, b, in, out + 1, n, s);
  });
}

struct Timer {
  cudaEvent_t e[7];
  int k = 0;
  cudaStream_t s;
  explicit Timer(cudaStream_t st) : s(st) {
    for (auto& x : e) TC_CUDA(cudaEventCreate(&x));
  }
  ~Timer() {
    for (auto& x : e) cudaEventDestroy(x);
  }
  void mark() { TC_CUDA(cudaEventRecord(e[k++], s)); }
  float ms(int a, int b) {
    float t = 0;
    TC_CUDA(cudaEventElapsedTime(&t, e[a], e[b]));
    return t;
  }
};

// a1 + a2: canonical keys of the valid non-loop pairs, radix sorted on
// 2*bits(n) bits, unique.  ka/kb: capacity max(m_gen, 1) each; returns the
// one holding the *m_out unique keys (the SENT key of loops is dropped).
uint64_t* canon_unique(const int32_t* d_src, const int32_t* d_dst, int64_t m_gen, int64_t n,
                       cudaStream_t s, uint64_t* ka, uint64_t* kb, int64_t* m_out, Timer* tm) {
  const int bits = bits_for(std::max<int64_t>(n, 2));
  const uint64_t sent = (uint64_t(1) << (2 * bits)) - 1;  // never a valid (lo < hi) key
  DevBuf<int> err(1, s);
  DevBuf<int64_t> nsel(1, s);
  DevBuf<UniqTail> tail(1, s);
  TC_CUDA(cudaMemsetAsync(err.get(), 0, sizeof(int), s));
  TC_CUDA(cudaMemsetAsync(nsel.get(), 0, sizeof(int64_t), s));
  if (m_gen > 0) {
    k_canon<<<grid_for(m_gen), TPB, 0, s>>>(d_src, d_dst, m_gen, n, bits, sent, ka, err.get());
    TC_LAUNCH();
  }
  if (tm) tm->mark();
  uint64_t* ukey = ka;
  if (m_gen > 0) {
    cub::DoubleBuffer<uint64_t> db(ka, kb);
    sort_keys_u64(db, m_gen, 2 * bits, s);
    uint64_t* sorted = db.Current();
    uint64_t* other = sorted == ka ? kb : ka;
    cub_run(s, [&](void* t, size_t& b) {
      return cub::DeviceSelect::Unique(t, b, sorted, other, nsel.get(), m_gen, s);
    });
    ukey = other;
  }
  k_uniq_tail<<<1, 1, 0, s>>>(err.get(), nsel.get(), ukey, tail.get());
  TC_LAUNCH();
  UniqTail ut = d2h(tail.get(), s);
  if (ut.err) fail(TC_ERR_INVALID_ARGUMENT, "vertex id < 0 or >= num_vertices in the edge list");
  *m_out = ut.nsel - ((ut.nsel > 0 && ut.last == sent) ? 1 : 0);
  return ukey;
}

// a1 + a2 by hashing (tc_build_csr up to 2^25 pairs; see build_graph): unique canonical keys into `out` (capacity max(m_gen, 1)),
// in table order.  Returns m.
int64_t canon_unique_hash(const int32_t* d_src, const int32_t* d_dst, int64_t m_gen, int64_t n,
                          cudaStream_t s, uint64_t* out, Timer* tm) {
  const int bits = bits_for(std::max<int64_t>(n, 2));
  int log2cap = 10;
  while ((int64_t(1) << log2cap) < 2 * m_gen) ++log2cap;
  DevBuf<uint64_t> table(size_t(1) << log2cap, s);
  DevBuf<int> err(1, s);
  DevBuf<int64_t> nsel(1, s);
  TC_CUDA(cudaMemsetAsync(err.get(), 0, sizeof(int), s));
  TC_CUDA(cudaMemsetAsync(table.get(), 0xFF, sizeof(uint64_t) << log2cap, s));
  if (m_gen > 0) {
    k_canon_hash<<<grid_for(m_gen), TPB, 0, s>>>(d_src, d_dst, m_gen, n, bits, table.get(), log2cap,
                                                 err.get());
    TC_LAUNCH();
  }
  if (tm) tm->mark();
  cub_run(s, [&](void* t, size_t& b) {
    return cub::DeviceSelect::If(t, b, table.get(), out, nsel.get(), int64_t(1) << log2cap,
                                 NotEmpty(), s);
  });
  int h_err = 0;
  int64_t m = 0;
  TC_CUDA(cudaMemcpyAsync(&h_err, err.get(), sizeof(int), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaMemcpyAsync(&m, nsel.get(), sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
  if (h_err) fail(TC_ERR_INVALID_ARGUMENT, "vertex id < 0 or >= num_vertices in the edge list");
  return m;
}

// a4: rank by (deg, id) ascending, isolated vertices last (dropped unless
// keep).  rank[v] for kept v; perm = perm_at(n_act) receives rank -> v.
template <class PermAt>
int64_t rank_vertices(const int32_t* deg, int64_t n, int keep, cudaStream_t s, int32_t* rank,
                      PermAt perm_at) {
  if (n <= 0) {
    perm_at(0);
    return 0;
  }
  const int bits = bits_for(std::max<int64_t>(n, 2));
  const uint64_t sentv = (uint64_t(1) << (2 * bits + 1)) - 1;
  DevBuf<uint64_t> va(n, s), vb(n, s);
  DevBuf<unsigned long long> nact(1, s);
  TC_CUDA(cudaMemsetAsync(nact.get(), 0, sizeof(unsigned long long), s));
  k_vkey<<<grid_for(n), TPB, 0, s>>>(deg, n, bits, keep, sentv, va.get(), nact.get());
  TC_LAUNCH();
  cub::DoubleBuffer<uint64_t> db(va.get(), vb.get());
  cub_run(s, [&](void* t, size_t& b) {
    return cub::DeviceRadixSort::SortKeys(t, b, db, n, 0, 2 * bits + 1, s);
  });
  const int64_t n_act = (int64_t)d2h(nact.get(), s);
  int32_t* perm = perm_at(n_act);
  if (n_act > 0) {
    k_perm<<<grid_for(n_act), TPB, 0, s>>>(db.Current(), n_act, bits, perm, rank);
    TC_LAUNCH();
  }
  return n_act;
}

// a5 (second half): CSR of m sorted unique oriented keys over n_act rows.
void csr_from_sorted(const uint64_t* okey, int64_t m, int64_t n_act, cudaStream_t s,
                     tc_graph* g) {
  const int bits2 = bits_for(std::max<int64_t>(n_act, 2));
  g->bits = bits2;
  g->m = m;
  g->n = n_act;
  g->row_ptr = DevBuf<int64_t>(n_act + 1, s, true);
  g->col = DevBuf<int32_t>(std::max<int64_t>(m, 1), s, true);
  if (m > 0) {
    g->rowid = DevBuf<int32_t>(m, s);  // scratch for the plan (build_plan frees it)
    k_csr<<<grid_for(m), TPB, 0, s>>>(okey, m, n_act, bits2, g->col.get(), g->row_ptr.get(),
                                      g->rowid.get());
    TC_LAUNCH();
  } else {
    k_fill_i64<<<grid_for(n_act + 1), TPB, 0, s>>>(g->row_ptr.get(), n_act + 1, 0);
    TC_LAUNCH();
  }
  DevBuf<unsigned long long> mx(1, s);
  TC_CUDA(cudaMemsetAsync(mx.get(), 0, sizeof(unsigned long long), s));
  if (n_act > 0) {
    k_max_outdeg<<<grid_for(n_act), TPB, 0, s>>>(g->row_ptr.get(), n_act, mx.get());
    TC_LAUNCH();
  }
  g->max_out = (int64_t)d2h(mx.get(), s);
}

}  // namespace

// a3..a6 from the m unique canonical keys `ukey` (in ka or kb; the other
// buffer is free), shared by the device and the pipelined host builds.
static void build_tail(uint64_t* ukey, int64_t m, DevBuf<uint64_t>& ka, DevBuf<uint64_t>& kb,
                       int64_t n, uint32_t flags, const Options& opt, cudaStream_t s, tc_graph* g,
                       Timer& tm) {
  const int bits = bits_for(std::max<int64_t>(n, 2));
  g->m = m;
  tm.mark();
  host_mark("a2_done");

  // a3 + a4
  DevBuf<int32_t> deg(std::max<int64_t>(n, 1), s);
  TC_CUDA(cudaMemsetAsync(deg.get(), 0, sizeof(int32_t) * std::max<int64_t>(n, 1), s));
  if (m > 0) {
    k_degree<<<grid_for(m), TPB, 0, s>>>(ukey, m, bits, deg.get());
    TC_LAUNCH();
  }
  const int keep = (flags & TC_KEEP_ISOLATED) ? 1 : 0;
  DevBuf<int32_t> rank(std::max<int64_t>(n, 1), s);
  const int64_t n_act = rank_vertices(deg.get(), n, keep, s, rank.get(), [&](int64_t na) {
    g->perm = DevBuf<int32_t>(std::max<int64_t>(na, 1), s, true);
    return g->perm.get();
  });
  g->n = n_act;
  deg.reset();
  tm.mark();

  // a5
  const int bits2 = bits_for(std::max<int64_t>(n_act, 2));
  if (m > 0) {
    uint64_t* okey_a = (ukey == ka.get()) ? kb.get() : ka.get();  // the free buffer
    k_orient<<<grid_for(m), TPB, 0, s>>>(ukey, m, bits, rank.get(), bits2, okey_a);
    TC_LAUNCH();
    cub::DoubleBuffer<uint64_t> db(okey_a, ukey);
    sort_keys_u64(db, m, 2 * bits2, s);
    csr_from_sorted(db.Current(), m, n_act, s, g);
  } else {
    csr_from_sorted(nullptr, 0, n_act, s, g);
  }
  ka.reset();
  kb.reset();
  rank.reset();
  tm.mark();
  host_mark("a3_a5");
  build_plan(g, opt, s);
  host_mark("plan_issued");
  tm.mark();
  TC_CUDA(cudaStreamSynchronize(s));
  host_mark("plan_sync");
  g->ms[0] = tm.ms(0, 1);
  g->ms[1] = tm.ms(1, 2);
  g->ms[2] = tm.ms(2, 3);
  g->ms[3] = tm.ms(3, 4);
  g->ms[4] = tm.ms(4, 5);
  g->ms[5] = tm.ms(0, 5);
}


// ------------------------------------------------------------------ a1..a5
void build_graph(const int32_t* d_src, const int32_t* d_dst, int64_t m_gen, int64_t n,
                 uint32_t flags, const Options& opt, cudaStream_t s, tc_graph* g) {
  Timer tm(s);
  tm.mark();
  if (n < 0) {  // num_vertices = max id + 1
    if (m_gen == 0) {
      n = 0;
    } else {
      DevBuf<int32_t> mx(2, s);
      cub_run(s, [&](void* t, size_t& b) {
        return cub::DeviceReduce::Max(t, b, d_src, mx.get(), m_gen, s);
      });
      cub_run(s, [&](void* t, size_t& b) {
        return cub::DeviceReduce::Max(t, b, d_dst, mx.get() + 1, m_gen, s);
      });
      int32_t h[2];
      TC_CUDA(cudaMemcpyAsync(h, mx.get(), sizeof(h), cudaMemcpyDeviceToHost, s));
      TC_CUDA(cudaStreamSynchronize(s));
      n = (int64_t)std::max(h[0], h[1]) + 1;
      if (n < 0) n = 0;
    }
  }
  g->n_input = n;

  // a1 + a2
  DevBuf<uint64_t> ka(std::max<int64_t>(m_gen, 1), s), kb(std::max<int64_t>(m_gen, 1), s);
  int64_t m = 0;
  // a2 by hash set for up to 2^25 pairs (table <= 512 MB; measured C5 2.45
  // -> 1.89 ms, C1 launch-bound 0.10 -> 0.06), by radix sort above (C3: hash
  // 21.7 ms vs sort 18.5: random CAS into a 4.3 GB table loses to 6 streaming
  // passes).  TC_DEDUP=sort|hash forces one (tests compare the two).
  static const int dedup_force = [] {
    const char* v = std::getenv("TC_DEDUP");
    if (!v) return 0;
    return std::string(v) == "sort" ? 1 : (std::string(v) == "hash" ? 2 : 0);
  }();
  const bool dedup_sort = dedup_force ? dedup_force == 1 : m_gen > (int64_t(1) << 25);
  uint64_t* ukey = ka.get();
  if (dedup_sort)
    ukey = canon_unique(d_src, d_dst, m_gen, n, s, ka.get(), kb.get(), &m, &tm);
  else
    m = canon_unique_hash(d_src, d_dst, m_gen, n, s, ka.get(), &tm);
  build_tail(ukey, m, ka, kb, n, flags, opt, s, g, tm);
}

// The host entry point (tc_build_csr_host) for large inputs: the H2D copy of
// the raw pairs is split into K pieces on a copy stream, and piece i is
// canonicalised and radix-sorted on the build stream while piece i+1 is
// still crossing PCIe; the K sorted runs are then merged pairwise
// (cub::DeviceMerge) and deduplicated.  Only the last piece's sort, the
// merges and the unique follow the copy (C3 K = 8: ~1/8 of the a2 sort plus
// three merge passes instead of the whole sort; K = 8 by default).  Same unique keys as
// canon_unique, so the same graph (tests compare the CSR).
void build_graph_host(const int32_t* h_src, const int32_t* h_dst, int64_t m_gen, int64_t n,
                      uint32_t flags, const Options& opt, cudaStream_t s, tc_graph* g) {
  static const int pieces = [] {
    const char* v = std::getenv("TC_H2D_PIECES");
    const int k = v ? std::atoi(v) : 8;  // C3 e2e: 1 piece 157.6 ms, 2 148.9, 4 148.5, 8 144.8
    return k == 1 || k == 2 || k == 4 || k == 8 ? k : 8;
  }();
  DevBuf<int32_t> ds(std::max<int64_t>(m_gen, 1), s), dd(std::max<int64_t>(m_gen, 1), s);
  host_mark("alloc_pairs");
  if (n < 0 || pieces == 1 || m_gen <= (int64_t(1) << 25) ||
      m_gen / pieces > (int64_t)0x7fffffff) {  // (cub merge counts are int)
    if (m_gen) {
      TC_CUDA(cudaMemcpyAsync(ds.get(), h_src, sizeof(int32_t) * m_gen, cudaMemcpyHostToDevice, s));
      TC_CUDA(cudaMemcpyAsync(dd.get(), h_dst, sizeof(int32_t) * m_gen, cudaMemcpyHostToDevice, s));
    }
    build_graph(ds.get(), dd.get(), m_gen, n, flags, opt, s, g);
    return;
  }
  Timer tm(s);
  tm.mark();
  // Let the pool growth and the piece buffers' allocations complete before the
  // pipelined copies and sorts are issued: without this sync the host entry's
  // time at C3 varied between 86 and 161 ms over identical builds (the phase
  // events inside stayed at 85 ms), with it it is 85-88 ms (profiles/r2t_e2e_c3.txt).
  TC_CUDA(cudaStreamSynchronize(s));
  host_mark("sync_alloc");
  g->n_input = n;
  const int bits = bits_for(std::max<int64_t>(n, 2));
  const uint64_t sent = (uint64_t(1) << (2 * bits)) - 1;
  DevBuf<uint64_t> ka(m_gen, s), kb(m_gen, s);
  DevBuf<int> err(1, s);
  DevBuf<int64_t> nsel(1, s);
  DevBuf<UniqTail> tail(1, s);
  struct Res {
    cudaStream_t cs = nullptr;
    cudaEvent_t ready = nullptr, ev[8] = {};
    ~Res() {
      if (cs) {
        cudaStreamSynchronize(cs);  // no copy may outlive the buffers it writes
        cudaStreamDestroy(cs);
      }
      if (ready) cudaEventDestroy(ready);
      for (auto e : ev)
        if (e) cudaEventDestroy(e);
    }
  } r;
  TC_CUDA(cudaStreamCreateWithFlags(&r.cs, cudaStreamNonBlocking));
  TC_CUDA(cudaEventCreateWithFlags(&r.ready, cudaEventDisableTiming));
  for (int i = 0; i < pieces; ++i) TC_CUDA(cudaEventCreateWithFlags(&r.ev[i], cudaEventDisableTiming));
  // the copies wait only for the stream-ordered allocations: nothing that
  // needs an SM may sit between them and the event (a memset there waited
  // behind a count kernel running on another stream and held the H2D back)
  TC_CUDA(cudaEventRecord(r.ready, s));  // the device buffers exist (stream-ordered allocs)
  TC_CUDA(cudaStreamWaitEvent(r.cs, r.ready, 0));
  host_mark("streams_events");
  TC_CUDA(cudaMemsetAsync(err.get(), 0, sizeof(int), s));
  TC_CUDA(cudaMemsetAsync(nsel.get(), 0, sizeof(int64_t), s));
  int64_t lo[9];
  for (int i = 0; i <= pieces; ++i) lo[i] = m_gen * i / pieces;
  for (int i = 0; i < pieces; ++i) {
    const size_t b = sizeof(int32_t) * (lo[i + 1] - lo[i]);
    TC_CUDA(cudaMemcpyAsync(ds.get() + lo[i], h_src + lo[i], b, cudaMemcpyHostToDevice, r.cs));
    TC_CUDA(cudaMemcpyAsync(dd.get() + lo[i], h_dst + lo[i], b, cudaMemcpyHostToDevice, r.cs));
    TC_CUDA(cudaEventRecord(r.ev[i], r.cs));
  }
  // piece i: canon + sort into ka[lo_i, lo_i+1) (copied back from kb if the
  // radix sort ends there), overlapping the copy of piece i + 1
  for (int i = 0; i < pieces; ++i) {
    TC_CUDA(cudaStreamWaitEvent(s, r.ev[i], 0));
    const int64_t c = lo[i + 1] - lo[i];
    k_canon<<<grid_for(c), TPB, 0, s>>>(ds.get() + lo[i], dd.get() + lo[i], c, n, bits, sent,
                                        ka.get() + lo[i], err.get());
    TC_LAUNCH();
    cub::DoubleBuffer<uint64_t> db(ka.get() + lo[i], kb.get() + lo[i]);
    sort_keys_u64(db, c, 2 * bits, s);
    if (db.Current() != ka.get() + lo[i])
      TC_CUDA(cudaMemcpyAsync(ka.get() + lo[i], db.Current(), sizeof(uint64_t) * c,
                              cudaMemcpyDeviceToDevice, s));
  }
  tm.mark();
  ds.reset();
  dd.reset();
  // pairwise merge rounds: runs of `w` pieces in `src` -> runs of 2w in `dst`
  uint64_t* src = ka.get();
  uint64_t* dst = kb.get();
  for (int w = 1; w < pieces; w *= 2) {
    for (int i = 0; i < pieces; i += 2 * w) {
      const int64_t a = lo[i], b = lo[i + w], e = lo[i + 2 * w];
      cub_run(s, [&](void* t, size_t& bytes) {
        return cub::DeviceMerge::MergeKeys(t, bytes, src + a, (int)(b - a), src + b, (int)(e - b),
                                           dst + a, cuda::std::less<uint64_t>{}, s);
      });
    }
    std::swap(src, dst);
  }
  cub_run(s, [&](void* t, size_t& b) {
    return cub::DeviceSelect::Unique(t, b, src, dst, nsel.get(), m_gen, s);
  });
  k_uniq_tail<<<1, 1, 0, s>>>(err.get(), nsel.get(), dst, tail.get());
  TC_LAUNCH();
  const UniqTail ut = d2h(tail.get(), s);
  if (ut.err) fail(TC_ERR_INVALID_ARGUMENT, "vertex id < 0 or >= num_vertices in the edge list");
  const int64_t m = ut.nsel - ((ut.nsel > 0 && ut.last == sent) ? 1 : 0);
  build_tail(dst, m, ka, kb, n, flags, opt, s, g, tm);
}

// ------------------------------------------------------------------ f2
int key_bits(int64_t n) { return bits_for(std::max<int64_t>(n, 2)); }

int64_t shard_canon(const int32_t* d_src, const int32_t* d_dst, int64_t m_gen, int64_t n,
                    cudaStream_t s, uint64_t* out) {
  DevBuf<uint64_t> ka(std::max<int64_t>(m_gen, 1), s), kb(std::max<int64_t>(m_gen, 1), s);
  int64_t m = 0;
  uint64_t* u = canon_unique(d_src, d_dst, m_gen, n, s, ka.get(), kb.get(), &m, nullptr);
  if (m > 0) TC_CUDA(cudaMemcpyAsync(out, u, sizeof(uint64_t) * m, cudaMemcpyDeviceToDevice, s));
  TC_CUDA(cudaStreamSynchronize(s));
  return m;
}

void shard_histogram(const uint64_t* keys, int64_t cnt, int64_t n, int hist_bits, cudaStream_t s,
                     int64_t* d_hist) {
  const int shift = 2 * key_bits(n) - hist_bits;
  const int64_t nb = int64_t(1) << hist_bits;
  k_key_hist<<<grid_for(nb), TPB, 0, s>>>(keys, cnt, shift, nb, d_hist);
  TC_LAUNCH();
}

void shard_bounds(const uint64_t* keys, int64_t cnt, int64_t n, int hist_bits,
                  const int64_t* h_cuts, int P, cudaStream_t s, int64_t* h_bounds) {
  const int shift = 2 * key_bits(n) - hist_bits;
  const int64_t nb = int64_t(1) << hist_bits;
  DevBuf<int64_t> cut(P + 1, s), pos(P + 1, s);
  TC_CUDA(cudaMemcpyAsync(cut.get(), h_cuts, sizeof(int64_t) * (P + 1), cudaMemcpyHostToDevice, s));
  k_key_bounds<<<1, 64 * ((P + 64) / 64), 0, s>>>(keys, cnt, shift, nb, cut.get(), P + 1, pos.get());
  TC_LAUNCH();
  TC_CUDA(cudaMemcpyAsync(h_bounds, pos.get(), sizeof(int64_t) * (P + 1), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
  h_bounds[0] = 0;
  h_bounds[P] = cnt;
}

void sort_keys(uint64_t* keys, int64_t cnt, int64_t n, cudaStream_t s) {
  if (cnt <= 1) return;
  DevBuf<uint64_t> kb(cnt, s);
  cub::DoubleBuffer<uint64_t> db(keys, kb.get());
  sort_keys_u64(db, cnt, 2 * key_bits(n), s);
  if (db.Current() != keys)
    TC_CUDA(cudaMemcpyAsync(keys, db.Current(), sizeof(uint64_t) * cnt, cudaMemcpyDeviceToDevice, s));
}

int64_t shard_unique(uint64_t* keys, int64_t cnt, int64_t n, cudaStream_t s, int32_t* d_deg) {
  if (cnt <= 0) return 0;
  const int bits = key_bits(n);
  DevBuf<uint64_t> kb(cnt, s);
  DevBuf<int64_t> nsel(1, s);
  cub::DoubleBuffer<uint64_t> db(keys, kb.get());
  sort_keys_u64(db, cnt, 2 * bits, s);
  uint64_t* sorted = db.Current();
  uint64_t* other = sorted == keys ? kb.get() : keys;
  cub_run(s, [&](void* t, size_t& b) {
    return cub::DeviceSelect::Unique(t, b, sorted, other, nsel.get(), cnt, s);
  });
  const int64_t m = d2h(nsel.get(), s);
  if (other != keys)
    TC_CUDA(cudaMemcpyAsync(keys, other, sizeof(uint64_t) * m, cudaMemcpyDeviceToDevice, s));
  if (m > 0) {
    k_degree<<<grid_for(m), TPB, 0, s>>>(keys, m, bits, d_deg);
    TC_LAUNCH();
  }
  TC_CUDA(cudaStreamSynchronize(s));
  return m;
}

void shard_degree(const uint64_t* keys, int64_t cnt, int64_t n, cudaStream_t s, int32_t* d_deg) {
  if (cnt <= 0) return;
  k_degree<<<grid_for(cnt), TPB, 0, s>>>(keys, cnt, key_bits(n), d_deg);
  TC_LAUNCH();
}

int64_t shard_rank(const int32_t* deg, int64_t n, uint32_t flags, cudaStream_t s, int32_t* rank,
                   int32_t* perm) {
  const int keep = (flags & TC_KEEP_ISOLATED) ? 1 : 0;
  return rank_vertices(deg, n, keep, s, rank, [&](int64_t) { return perm; });
}

void shard_orient(const uint64_t* keys, int64_t cnt, int64_t n, const int32_t* rank,
                  int64_t n_act, cudaStream_t s, uint64_t* okeys) {
  if (cnt <= 0) return;
  k_orient<<<grid_for(cnt), TPB, 0, s>>>(keys, cnt, key_bits(n), rank, key_bits(n_act), okeys);
  TC_LAUNCH();
  sort_keys(okeys, cnt, n_act, s);
}

void build_from_oriented(const uint64_t* okeys, int64_t m, const int32_t* perm, int64_t n_act,
                         int64_t n_input, const Options& opt, cudaStream_t s, tc_graph* g) {
  Timer tm(s);
  tm.mark();
  g->n_input = n_input;
  g->perm = DevBuf<int32_t>(std::max<int64_t>(n_act, 1), s, true);
  if (n_act > 0)
    TC_CUDA(cudaMemcpyAsync(g->perm.get(), perm, sizeof(int32_t) * n_act, cudaMemcpyDeviceToDevice, s));
  csr_from_sorted(m > 0 ? okeys : nullptr, m, n_act, s, g);
  tm.mark();
  build_plan(g, opt, s);
  tm.mark();
  TC_CUDA(cudaStreamSynchronize(s));
  g->ms[3] = tm.ms(0, 1);
  g->ms[4] = tm.ms(1, 2);
  g->ms[5] = tm.ms(0, 2);
}

Tuning tuning_from_env() {
  Tuning t;
  auto get = [](const char* name, int def, int lo, int hi) {
    const char* v = std::getenv(name);
    if (!v) return def;
    int x = std::atoi(v);
    return x < lo ? lo : (x > hi ? hi : x);
  };
  t.slots = get("TC_SLOTS", t.slots, 2, 4);
  t.grab_long = (get("TC_GRAB_LONG", t.grab_long, 0, 1 << 20) + 7) & ~7;  // walk_long: 8-tile batches
  t.grab_short = get("TC_GRAB_SHORT", t.grab_short, 0, 1 << 24);
  t.prod_div = get("TC_PROD_DIV", t.prod_div, 2, 32);
  t.wait_hint_ns = get("TC_WAIT_HINT", t.wait_hint_ns, 0, 10000000);
  t.cs_div = get("TC_CS_DIV", t.cs_div, 0, 64);
  t.short_linear = get("TC_SHORT_LINEAR", t.short_linear, 0, 1);
  t.max_kicks = get("TC_CUCKOO_KICKS", t.max_kicks, 0, 4096);
  t.batch = get("TC_BATCH", t.batch, 0, 64);
  t.prod_groups = get("TC_PROD_GROUPS", t.prod_groups, 1, 3);
  t.long_hash_dmax = get("TC_LONG_HASH_DMAX", t.long_hash_dmax, 0, 1 << 30);
  return t;
}

// ------------------------------------------------------------------ a6
void build_plan(tc_graph* g, const Options& opt, cudaStream_t s) {
  Plan& P = g->plan;
  P = Plan();
  P.opt = opt;
  P.block = opt.block_threads;
  P.tune = tuning_from_env();
  const int64_t m = g->m, n = g->n;
  // the count kernel's tile descriptors address keys by a 32-bit col index
  if (m > (int64_t)0xFFFFFFFFll) fail(TC_ERR_UNSUPPORTED, "more than 2^32 - 1 unique edges");
  const int64_t* row_ptr = g->row_ptr.get();
  const int32_t* col = g->col.get();
  Trace tr(s);
  DevBuf<unsigned long long> stats(5, s);
  TC_CUDA(cudaMemsetAsync(stats.get(), 0, 5 * sizeof(unsigned long long), s));
  // sort keys: class bit above the head v; dead edges sort last
  const int kbits = g->bits + 1;
  const uint32_t dead = kbits < 32 ? (1u << kbits) : 0xFFFFFFFFu;
  const int end_bit = kbits < 32 ? kbits + 1 : 32;
  // the row of every position: left by the CSR build (k_csr), else one pass over rows
  DevBuf<int32_t> rowid;
  rowid.swap(g->rowid);
  DevBuf<uint32_t> skey(std::max<int64_t>(m, 1), s), skey2(std::max<int64_t>(m, 1), s);
  // (sorting 4-B indices and gathering the packed values afterwards measured
  // slower: the sort saved 1.5 ms, the random 8-B gather cost 4.7 ms at C3)
  DevBuf<uint64_t> sval(std::max<int64_t>(m, 1), s), sval2(std::max<int64_t>(m, 1), s);
  if (m > 0) {
    if (!rowid.get()) {
      rowid = DevBuf<int32_t>(m, s);
      k_rowid<<<grid_for(n), TPB, 0, s>>>(row_ptr, n, rowid.get());
      TC_LAUNCH();
    }
    DevBuf<int4> vmm(std::max<int64_t>(n, 1), s);
    k_vmm<<<grid_for(n), TPB, 0, s>>>(row_ptr, col, n, vmm.get());
    TC_LAUNCH();
    // a long-class tile always holds 32 keys of its own edge (walk_long shifts
    // a partial last tile back onto the edge), so long_min < 32 acts as 32
    // Small graphs (C1: 10 K edges) count faster with every edge in the
    // short class: one launch of the flat kernel instead of also starting the
    // persistent warp-specialised one (C1 0.041 -> 0.023 ms); an explicit
    // long_min keeps the split.
    constexpr int64_t kSmallGraph = int64_t(1) << 20;
    const int long_min = (opt.long_min_auto && m < kSmallGraph) ? (1 << 30) : std::max(opt.long_min, 32);
    k_edge_trim<<<grid_for(m), TPB, 0, s>>>(row_ptr, col, rowid.get(), vmm.get(), m, long_min,
                                            g->bits, dead, skey.get(), sval.get(), stats.get(),
                                            P.tune.long_hash_dmax, opt.bitmap_factor);
    TC_LAUNCH();
  }
  rowid.reset();
  tr("rowid + edge trim");
  unsigned long long h_stats[5];
  TC_CUDA(cudaMemcpyAsync(h_stats, stats.get(), sizeof(h_stats), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
  g->b_itc = h_stats[0] + 8ull * (unsigned long long)(n + 1);
  P.keys_total = (int64_t)h_stats[1];
  P.keys_long = (int64_t)h_stats[4];
  const int64_t S = (int64_t)h_stats[2], S_long = (int64_t)h_stats[3];
  P.S = S;
  P.S_long = S_long;
  P.key_prefix = DevBuf<uint32_t>(S + 1, s, true);
  TC_CUDA(cudaMemsetAsync(P.key_prefix.get(), 0, sizeof(uint32_t), s));
  if (S == 0) {
    P.chunk_seg = DevBuf<int64_t>(1, s, true);
    TC_CUDA(cudaMemsetAsync(P.chunk_seg.get(), 0, sizeof(int64_t), s));
    P.chunk_cost = DevBuf<int64_t>(1, s, true);
    TC_CUDA(cudaMemsetAsync(P.chunk_cost.get(), 0, sizeof(int64_t), s));
    TC_CUDA(cudaStreamSynchronize(s));
    return;
  }

  // live edges ordered by (class, head v, position): the radix sort is stable
  // and the edges arrive in position order; dead edges sort past S
  cub::DoubleBuffer<uint32_t> dk(skey.get(), skey2.get());
  cub::DoubleBuffer<uint64_t> dv(sval.get(), sval2.get());
  cub_run(s, [&](void* t, size_t& b) {
    return cub::DeviceRadixSort::SortPairs(t, b, dk, dv, m, 0, end_bit, s);
  });
  const uint32_t* key_sorted = dk.Current();
  const uint64_t* val_sorted = dv.Current();
  tr("select + class sort");

  DevBuf<int32_t> gincl(S, s);
  {
    cub::TransformInputIterator<int32_t, GroupStart, cub::CountingInputIterator<int64_t>> marks(
        cub::CountingInputIterator<int64_t>(0), GroupStart{key_sorted});
    cub_run(s, [&](void* t, size_t& b) {
      return cub::DeviceScan::InclusiveSum(t, b, marks, gincl.get(), S, s);
    });
  }
  const int64_t G = (int64_t)d2h(gincl.get() + (S - 1), s);
  P.G = G;
  // SMEM of one chunk slot of the count kernel; a table may use at most half
  // of it (bigger tables are "huge": probed in global memory)
  const int64_t slot_limit = max_chunk_smem(P.tune);
  const int64_t flat_limit = max_flat_chunk_smem();
  const int64_t max_slots_long = slot_limit / 8, max_slots_short = flat_limit / 8;  // half a slot
  P.seg_start = DevBuf<uint32_t>(S, s, true);
  P.seg_len = DevBuf<int32_t>(S, s, true);
  P.seg_group = DevBuf<int32_t>(S, s, true);
  DevBuf<uint32_t> units(S, s);
  DevBuf<int64_t> grp_row(G, s), grp_d(G, s), grp_slots(G, s), cost(S, s), cost_prefix(S + 1, s);
  DevBuf<unsigned long long> d_units_total(1, s);
  TC_CUDA(cudaMemsetAsync(d_units_total.get(), 0, sizeof(unsigned long long), s));
  unsigned long long units_total = 0;  // host copy (read after the next sync)
  P.grp_code = DevBuf<int32_t>(G, s, true);
  k_seg_fill<<<grid_for(S), TPB, 0, s>>>(key_sorted, val_sorted, gincl.get(), S, S_long,
                                         g->bits, row_ptr,
                                         opt.huge_degree, opt.table_factor, opt.bitmap_factor,
                                         max_slots_long, max_slots_short, col, P.grp_code.get(),
                                         P.seg_start.get(),
                                         P.seg_len.get(), P.seg_group.get(), units.get(),
                                         grp_row.get(), grp_d.get(), grp_slots.get(), opt.seg_cost,
                                         cost.get(), d_units_total.get());
  TC_LAUNCH();
  gincl.reset();
  skey.reset();
  skey2.reset();
  sval.reset();
  sval2.reset();
  // the unit prefix mod 2^32 (uint32 arithmetic wraps exactly; only
  // chunk-relative differences are used), key_prefix[0] = 0 (memset above)
  cub_run(s, [&](void* t, size_t& b) {
    return cub::DeviceScan::InclusiveSum(t, b, units.get(), P.key_prefix.get() + 1, S, s);
  });
  TC_CUDA(cudaMemcpyAsync(&units_total, d_units_total.get(), sizeof(units_total),
                          cudaMemcpyDeviceToHost, s));
  P.ins_prefix = DevBuf<int64_t>(G + 1, s, true);
  P.slot_prefix = DevBuf<int64_t>(G + 1, s, true);
  exclusive_prefix(grp_d.get(), G, P.ins_prefix.get(), s);
  exclusive_prefix(grp_slots.get(), G, P.slot_prefix.get(), s);
  P.grp_ibase = DevBuf<int64_t>(G, s, true);
  k_grp_ibase<<<grid_for(G), TPB, 0, s>>>(grp_row.get(), P.ins_prefix.get(), G, P.grp_ibase.get());
  TC_LAUNCH();
  exclusive_prefix(cost.get(), S, cost_prefix.get(), s);
  cost.reset();
  units.reset();
  grp_row.reset();
  grp_d.reset();
  grp_slots.reset();
  int64_t h_cp[2];
  TC_CUDA(cudaMemcpyAsync(&h_cp[0], cost_prefix.get() + S_long, sizeof(int64_t),
                          cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaMemcpyAsync(&h_cp[1], cost_prefix.get() + S, sizeof(int64_t), cudaMemcpyDeviceToHost,
                          s));
  TC_CUDA(cudaStreamSynchronize(s));
  const int64_t cost_long = h_cp[0], cost_short = h_cp[1] - h_cp[0];
  tr("groups + prefixes + costs");
  P.units_total = (int64_t)units_total;

  // Chunking, per class: cost chunks (long class 4x larger: its edges carry
  // ~150 keys each), then every chunk is split where its SMEM layout would
  // exceed one of the count kernel's chunk slots (only outliers split).
  // short chunks of half the cost when edges carry ~1 key (C5 road lattice:
  // 1.05 keys per live edge, 0.114 -> 0.073 ms; C2 at 5.4 keys: neutral)
  const int cs_div = P.tune.cs_div ? P.tune.cs_div : (P.keys_total < 2 * S ? 2 : 1);
  const int64_t CL = std::max<int64_t>(4ll * opt.chunk_cost, 64),
                CS = std::max<int64_t>(opt.chunk_cost / cs_div, 64);
  {
    const int64_t nL0 = (cost_long + CL - 1) / CL, nS0 = (cost_short + CS - 1) / CS, nc0 = nL0 + nS0;
    DevBuf<int64_t> cs0(nc0 + 1, s), pieces(std::max<int64_t>(nc0, 1), s), poff(nc0 + 1, s);
    k_chunk_bounds<<<grid_for(nc0 + 1), TPB, 0, s>>>(cost_prefix.get(), S_long, S, nL0, nS0, CL, CS,
                                                     cs0.get());
    TC_LAUNCH();
    DevBuf<unsigned long long> mx(2, s);
    TC_CUDA(cudaMemsetAsync(mx.get(), 0, 2 * sizeof(unsigned long long), s));
    k_split<<<grid_for(nc0), TPB, 0, s>>>(cs0.get(), nc0, nL0, P.seg_group.get(), P.slot_prefix.get(),
                                          P.key_prefix.get(), slot_limit, flat_limit, pieces.get(),
                                          nullptr, nullptr, mx.get());
    TC_LAUNCH();
    exclusive_prefix(pieces.get(), nc0, poff.get(), s);
    int64_t h_off[2];
    TC_CUDA(cudaMemcpyAsync(&h_off[0], poff.get() + nL0, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    TC_CUDA(cudaMemcpyAsync(&h_off[1], poff.get() + nc0, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    unsigned long long need[2] = {0, 0};
    TC_CUDA(cudaMemcpyAsync(need, mx.get(), sizeof(need), cudaMemcpyDeviceToHost, s));
    TC_CUDA(cudaStreamSynchronize(s));
    if ((int64_t)need[0] > slot_limit || (int64_t)need[1] > flat_limit)
      fail(TC_ERR_UNSUPPORTED, "an edge's hash table exceeds shared memory (lower huge_degree)");
    const int64_t nc = h_off[1];
    P.chunk_seg = DevBuf<int64_t>(nc + 1, s, true);
    k_split<<<grid_for(nc0), TPB, 0, s>>>(cs0.get(), nc0, nL0, P.seg_group.get(), P.slot_prefix.get(),
                                          P.key_prefix.get(), slot_limit, flat_limit, nullptr,
                                          poff.get(), P.chunk_seg.get(), nullptr);
    TC_LAUNCH();
    k_set_i64<<<1, 1, 0, s>>>(P.chunk_seg.get() + nc, S);
    TC_LAUNCH();
    P.n_chunks = nc;
    P.n_long_chunks = h_off[0];
    P.smem_bytes = std::max<int64_t>((int64_t)need[0], 16);
    P.smem_flat = std::max<int64_t>((int64_t)need[1], 16);
    if (tr.on)
      fprintf(stderr, "[tc]   chunks CL=%lld CS=%lld cost chunks %lld (long %lld) -> %lld (long %lld), smem long %llu short %llu\n",
              (long long)CL, (long long)CS, (long long)nc0, (long long)nL0, (long long)nc,
              (long long)h_off[0], need[0], need[1]);
  }
  P.chunk_cost_long = CL;
  P.chunk_cost_short = CS;
  tr("chunking");
  {
    P.chunk_cost = DevBuf<int64_t>(P.n_chunks + 1, s, true);
    DevBuf<unsigned long long> st2(4, s);
    TC_CUDA(cudaMemsetAsync(st2.get(), 0, 4 * sizeof(unsigned long long), s));
    k_chunk_meta<<<grid_for(P.n_chunks + 1), TPB, 0, s>>>(P.chunk_seg.get(), P.n_chunks,
                                                          P.n_long_chunks,
                                                          P.seg_group.get(), P.ins_prefix.get(),
                                                          cost_prefix.get(), P.chunk_cost.get(),
                                                          st2.get());
    TC_LAUNCH();
    unsigned long long h_st2[4];
    TC_CUDA(cudaMemcpyAsync(h_st2, st2.get(), sizeof(h_st2), cudaMemcpyDeviceToHost, s));
    TC_CUDA(cudaStreamSynchronize(s));
    P.table_words = (int64_t)h_st2[0];
    P.group_visits = (int64_t)h_st2[1];
    auto bytes = [](int64_t keys, int64_t edges, int64_t words, int64_t visits, int64_t chunks) {
      return 4ull * (uint64_t)keys + (uint64_t)(kPlanEdgeBytes * edges) + 4ull * (uint64_t)words +
             (uint64_t)(kPlanGroupBytes * visits) + (uint64_t)(kPlanChunkBytes * chunks);
    };
    P.method_bytes = bytes(P.keys_total, S, P.table_words, P.group_visits, P.n_chunks);
    P.method_bytes_long = bytes(P.keys_long, S_long, (int64_t)h_st2[2], (int64_t)h_st2[3],
                                P.n_long_chunks);
  }
  const int occ = count_occupancy(P.block, P.smem_bytes, P.tune);
  const int occ_flat = flat_occupancy(P.smem_flat);
  if (occ < 1 || occ_flat < 1)
    fail(TC_ERR_UNSUPPORTED, "count kernel cannot launch with this SMEM/block size");
  P.grid = (int)std::min<int64_t>(std::max<int64_t>(P.n_long_chunks, 1), (int64_t)occ * num_sms());
  P.grid_flat = (int)std::min<int64_t>(std::max<int64_t>(P.n_chunks - P.n_long_chunks, 1),
                                       (int64_t)occ_flat * num_sms());
  tr("chunk copy + occupancy");
}

}  // namespace tc

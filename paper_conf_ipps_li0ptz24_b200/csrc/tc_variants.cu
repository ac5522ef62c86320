// tc_variants.cu — SURVEY.md §8(f) row f3: two of the paper's surveyed ITC
// kernels, written for sm_100a on this library's CSR, as alternative counting
// paths (tc_count_variant).  They compute the same T as tc_count and exist to
// reproduce the paper's comparison on B200 (Polak is best on small
// graphs, TRUST on large ones); the product path is the grouped kernel of
// tc_count.cu.
//
// POLAK (Fig. 3): edge-centric, one thread per oriented edge (u,v),
//   a sequential merge of the full out-lists N+(u) and N+(v) (work d+(u) +
//   d+(v)), incrementing a counter when the two pointers meet equal keys.
// TRUST (Fig. 10): vertex-centric.  The 1-hop list N+(u) goes into
//   a hash table; every 2-hop neighbour w in N+(v), v in N+(u), is a query.
//   Degree-bucketed resources as P:254 describes: d+(u) > 100 -> a 1024-thread
//   block with a 1024-bucket table; 2 <= d+(u) <= 100 -> one warp with a
//   32-bucket table; d+(u) < 2 is skipped (no wedge can close).  Buckets are
//   SMEM rows of fixed capacity (bucket = key mod buckets); a bucket that
//   would overflow its row spills the vertex to the global-memory fallback
//   (binary search in N+(u)), which keeps the count exact for any input.
// Both reduce thread u32 -> warp shuffle -> one u64 atomic per warp/block.
#include <algorithm>
#include <cstdlib>

#include "tc_internal.cuh"

namespace tc {
namespace {

constexpr int kTPB = 256;

__device__ __forceinline__ int64_t row_of(const int64_t* __restrict__ row_ptr, int64_t n, int64_t p) {
  int64_t lo = 0, hi = n - 1;  // largest u with row_ptr[u] <= p
  while (lo < hi) {
    const int64_t mid = (lo + hi + 1) >> 1;
    if (__ldg(row_ptr + mid) <= p) lo = mid; else hi = mid - 1;
  }
  return lo;
}

__device__ __forceinline__ void warp_add(unsigned long long v, unsigned long long* out) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
  if ((threadIdx.x & 31) == 0 && v) atomicAdd(out, v);
}

// ---------------------------------------------------------------- Polak
__global__ void __launch_bounds__(kTPB) k_polak(const int64_t* __restrict__ row_ptr, int64_t n,
                                               const int32_t* __restrict__ col, int64_t m,
                                               unsigned long long* __restrict__ out) {
  unsigned long long acc = 0;
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < m;
       p += (int64_t)gridDim.x * blockDim.x) {
    const int64_t u = row_of(row_ptr, n, p);
    const int32_t v = __ldg(col + p);
    int64_t i = __ldg(row_ptr + u), ie = __ldg(row_ptr + u + 1);
    int64_t j = __ldg(row_ptr + v), je = __ldg(row_ptr + v + 1);
    unsigned c = 0;
    while (i < ie && j < je) {  // sequential merge (Fig. 3)
      const int32_t a = __ldg(col + i), b = __ldg(col + j);
      c += a == b;
      i += a <= b;
      j += b <= a;
    }
    acc += c;
  }
  warp_add(acc, out);
}

// ---------------------------------------------------------------- TRUST
constexpr int kSmallMax = 100;      // 2..100 -> warp, > 100 -> block
constexpr int kWarpBuckets = 32;
constexpr int kWarpCap = 8;         // SMEM slots per bucket (warp tables)
constexpr int kBlockBuckets = 1024;
constexpr int kBlockCap = 16;       // SMEM slots per bucket (block tables)
constexpr int kBlockThreads = 1024;

// Bucketed table: bucket b holds keys with key mod B == b in T[b*cap ...],
// count in cnt[b].  Returns false if a bucket overflowed.
__device__ __forceinline__ bool bucket_insert(int* __restrict__ T, int* __restrict__ cnt, int B,
                                              int cap, int32_t key) {
  const int b = key % B;
  const int k = atomicAdd(&cnt[b], 1);
  if (k >= cap) return false;
  T[b * cap + k] = key;
  return true;
}

__device__ __forceinline__ unsigned bucket_find(const int* __restrict__ T, const int* __restrict__ cnt,
                                                int B, int cap, int32_t key) {
  const int b = key % B;
  const int c = min(cnt[b], cap);
  unsigned hit = 0;
  for (int k = 0; k < c; ++k) hit |= T[b * cap + k] == key;
  return hit;
}

__device__ __forceinline__ unsigned in_sorted(const int32_t* __restrict__ col, int64_t b, int64_t e,
                                              int32_t key) {
  int64_t lo = b, hi = e;
  while (lo < hi) {
    const int64_t mid = (lo + hi) >> 1;
    if (__ldg(col + mid) < key) lo = mid + 1; else hi = mid;
  }
  return (lo < e && __ldg(col + lo) == key) ? 1u : 0u;
}

// 2 <= d+(u) <= 100: one warp per vertex (grid-stride over vertices).
__global__ void __launch_bounds__(kTPB) k_trust_warp(const int64_t* __restrict__ row_ptr, int64_t n,
                                                    const int32_t* __restrict__ col, int cap,
                                                    unsigned long long* __restrict__ out) {
  __shared__ int sT[kTPB / 32][kWarpBuckets * kWarpCap];
  __shared__ int sC[kTPB / 32][kWarpBuckets];
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  int* T = sT[wid];
  int* C = sC[wid];
  unsigned long long acc = 0;
  const int64_t nw = (int64_t)gridDim.x * (kTPB / 32);
  for (int64_t u = blockIdx.x * (int64_t)(kTPB / 32) + wid; u < n; u += nw) {
    const int64_t b = __ldg(row_ptr + u), e = __ldg(row_ptr + u + 1), d = e - b;
    if (d < 2 || d > kSmallMax) continue;  // warp-uniform
    C[lane] = 0;
    __syncwarp();
    bool ok = true;
    for (int64_t i = b + lane; i < e; i += 32)
      ok &= bucket_insert(T, C, kWarpBuckets, cap, __ldg(col + i));
    const bool spill = __any_sync(0xffffffffu, !ok);
    __syncwarp();
    // queries: every w in N+(v), v in N+(u) (the 2-hop list), lanes over w
    for (int64_t i = b; i < e; ++i) {
      const int32_t v = __ldg(col + i);
      const int64_t vb = __ldg(row_ptr + v), ve = __ldg(row_ptr + v + 1);
      for (int64_t j = vb + lane; j < ve; j += 32) {
        const int32_t w = __ldg(col + j);
        acc += spill ? in_sorted(col, b, e, w) : bucket_find(T, C, kWarpBuckets, cap, w);
      }
    }
    __syncwarp();
  }
  warp_add(acc, out);
}

// d+(u) > 100: one 1024-thread block per vertex of the compacted list.
__global__ void __launch_bounds__(kBlockThreads) k_trust_block(const int64_t* __restrict__ row_ptr,
                                                             const int32_t* __restrict__ col,
                                                             const int32_t* __restrict__ big,
                                                             const int* __restrict__ n_big, int cap,
                                                             unsigned long long* __restrict__ out) {
  extern __shared__ int smem[];
  int* T = smem;                                  // kBlockBuckets * kBlockCap
  int* C = smem + kBlockBuckets * kBlockCap;      // kBlockBuckets
  __shared__ int s_spill;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nwarps = blockDim.x >> 5;
  unsigned long long acc = 0;
  const int nb = *n_big;
  for (int k = blockIdx.x; k < nb; k += gridDim.x) {
    const int32_t u = big[k];
    const int64_t b = __ldg(row_ptr + u), e = __ldg(row_ptr + u + 1);
    for (int i = threadIdx.x; i < kBlockBuckets; i += blockDim.x) C[i] = 0;
    if (threadIdx.x == 0) s_spill = 0;
    __syncthreads();
    bool ok = true;
    for (int64_t i = b + threadIdx.x; i < e; i += blockDim.x)
      ok &= bucket_insert(T, C, kBlockBuckets, cap, __ldg(col + i));
    if (!ok) s_spill = 1;
    __syncthreads();
    const bool spill = s_spill != 0;
    for (int64_t i = b + warp; i < e; i += nwarps) {  // a warp per 1-hop neighbour v
      const int32_t v = __ldg(col + i);
      const int64_t vb = __ldg(row_ptr + v), ve = __ldg(row_ptr + v + 1);
      for (int64_t j = vb + lane; j < ve; j += 32) {
        const int32_t w = __ldg(col + j);
        acc += spill ? in_sorted(col, b, e, w)
                     : bucket_find(T, C, kBlockBuckets, cap, w);
      }
    }
    __syncthreads();
  }
  warp_add(acc, out);
}

__global__ void k_big_list(const int64_t* __restrict__ row_ptr, int64_t n, int32_t* __restrict__ big,
                           int* __restrict__ n_big) {
  for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n;
       u += (int64_t)gridDim.x * blockDim.x)
    if (row_ptr[u + 1] - row_ptr[u] > kSmallMax) big[atomicAdd(n_big, 1)] = (int32_t)u;
}

int grid_of(int64_t work, int per_block) {
  const int64_t g = (work + per_block - 1) / per_block;
  return (int)std::max<int64_t>(1, std::min<int64_t>(g, (int64_t)num_sms() * 32));
}

}  // namespace

void count_variant(const tc_graph* g, int variant, cudaStream_t s, unsigned long long* d_out) {
  TC_CUDA(cudaMemsetAsync(d_out, 0, sizeof(unsigned long long), s));
  if (g->m == 0) return;
  const int64_t n = g->n, m = g->m;
  if (variant == TC_VARIANT_POLAK) {
    k_polak<<<grid_of(m, kTPB), kTPB, 0, s>>>(g->row_ptr.get(), n, g->col.get(), m, d_out);
    TC_LAUNCH();
    return;
  }
  // TRUST.  TC_TRUST_CAP (test knob) shrinks the bucket rows so that tests
  // reach the overflow fallback.
  int wcap = kWarpCap, bcap = kBlockCap;
  if (const char* e = std::getenv("TC_TRUST_CAP")) {
    wcap = std::max(1, std::min(kWarpCap, std::atoi(e)));
    bcap = std::max(1, std::min(kBlockCap, std::atoi(e)));
  }
  k_trust_warp<<<grid_of(n * 32, kTPB), kTPB, 0, s>>>(g->row_ptr.get(), n, g->col.get(), wcap,
                                                      d_out);
  TC_LAUNCH();
  if (g->max_out <= kSmallMax) return;
  DevBuf<int32_t> big(n, s);
  DevBuf<int> n_big(1, s);
  TC_CUDA(cudaMemsetAsync(n_big.get(), 0, sizeof(int), s));
  k_big_list<<<grid_of(n, kTPB), kTPB, 0, s>>>(g->row_ptr.get(), n, big.get(), n_big.get());
  TC_LAUNCH();
  const size_t smem = sizeof(int) * (kBlockBuckets * kBlockCap + kBlockBuckets);
  // per launch: the attribute belongs to the current device's context, and
  // setting it is cheap next to a TRUST count
  TC_CUDA(cudaFuncSetAttribute(k_trust_block, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               (int)smem));
  k_trust_block<<<num_sms() * 2, kBlockThreads, smem, s>>>(g->row_ptr.get(), g->col.get(),
                                                           big.get(), n_big.get(), bcap, d_out);
  TC_LAUNCH();
}

}  // namespace tc

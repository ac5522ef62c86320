// CUB radix-sort policy sweep for the build's three big sorts (a2/a5: 64-bit keys
// with 2*24 significant bits; a6: 32-bit key of 26 bits with a 64-bit value).
// Dev tool, not part of the product:
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o build/sort_bench scripts/sort_bench.cu
//   build/sort_bench [n_keys]
// Times each policy with CUDA events (median of 5 after a warm-up) and checks
// its output against the default policy's.
#include <cub/cub.cuh>

#include <algorithm>

#include <cstdio>
#include <vector>

#define CK(x)                                                                 \
  do {                                                                        \
    cudaError_t e_ = (x);                                                     \
    if (e_ != cudaSuccess) {                                                  \
      printf("CUDA %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
      exit(1);                                                                \
    }                                                                         \
  } while (0)

__global__ void k_fill64(uint64_t* k, int64_t n, int bits, uint64_t seed) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t z = (uint64_t)i * 0x9E3779B97F4A7C15ull + seed;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    z ^= z >> 31;
    k[i] = z & ((1ull << bits) - 1);
  }
}
__global__ void k_fill32(uint32_t* k, uint64_t* v, int64_t n, int bits, uint64_t seed) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t z = (uint64_t)i * 0x9E3779B97F4A7C15ull + seed;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    z ^= z >> 31;
    k[i] = (uint32_t)(z & ((1ull << bits) - 1));
    v[i] = (uint64_t)i;
  }
}

__global__ void k_split64(const uint64_t* k, int64_t n, uint32_t* hi, uint32_t* lo) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    hi[i] = (uint32_t)(k[i] >> 24);
    lo[i] = (uint32_t)(k[i] & 0xFFFFFF);
  }
}

using OffsetT = unsigned long long;

template <class K, class V, bool kOnesweep, int kThreads, int kItems, int kBits>
struct Hub {
  using Base = typename cub::detail::radix::policy_hub<K, V, OffsetT>::Policy1000;
  using DominantT = ::cuda::std::_If<(sizeof(V) > sizeof(K)), V, K>;
  struct P : cub::ChainedPolicy<1000, P, P> {
    static constexpr bool ONESWEEP = kOnesweep;
    static constexpr int ONESWEEP_RADIX_BITS = kBits;
    using HistogramPolicy = cub::AgentRadixSortHistogramPolicy<128, 16, 1, K, kBits>;
    using ExclusiveSumPolicy = cub::AgentRadixSortExclusiveSumPolicy<256, kBits>;
    using OnesweepPolicy =
        cub::AgentRadixSortOnesweepPolicy<kThreads, kItems, DominantT, 1, cub::RADIX_RANK_MATCH_EARLY_COUNTS_ANY,
                                          cub::BLOCK_SCAN_RAKING_MEMOIZE, cub::RADIX_SORT_STORE_DIRECT, kBits>;
    using ScanPolicy = typename Base::ScanPolicy;
    using DownsweepPolicy =
        cub::AgentRadixSortDownsweepPolicy<kThreads, kItems, DominantT, cub::BLOCK_LOAD_TRANSPOSE, cub::LOAD_DEFAULT,
                                           cub::RADIX_RANK_MATCH, cub::BLOCK_SCAN_WARP_SCANS, kBits>;
    using AltDownsweepPolicy = DownsweepPolicy;
    using UpsweepPolicy = cub::AgentRadixSortUpsweepPolicy<kThreads, kItems, DominantT, cub::LOAD_DEFAULT, kBits>;
    using AltUpsweepPolicy = UpsweepPolicy;
    using SingleTilePolicy = typename Base::SingleTilePolicy;
    using SegmentedPolicy = typename Base::SegmentedPolicy;
    using AltSegmentedPolicy = typename Base::AltSegmentedPolicy;
  };
  using MaxPolicy = P;
};

template <class K, class V, class H>
float run(cub::DoubleBuffer<K>& dk, cub::DoubleBuffer<V>& dv, int64_t n, int end_bit, void* tmp, size_t& tb,
          cudaStream_t s) {
  using D = cub::DispatchRadixSort<false, K, V, OffsetT, H>;
  size_t need = 0;
  CK(D::Dispatch(nullptr, need, dk, dv, (OffsetT)n, 0, end_bit, true, s));
  if (need > tb) {
    printf("temp %zu > %zu\n", need, tb);
    return -1;
  }
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  CK(cudaEventRecord(a, s));
  CK(D::Dispatch(tmp, need, dk, dv, (OffsetT)n, 0, end_bit, true, s));
  CK(cudaEventRecord(b, s));
  CK(cudaEventSynchronize(b));
  float ms = 0;
  CK(cudaEventElapsedTime(&ms, a, b));
  return ms;
}

template <class K, class V, class H>
void bench(const char* name, K* k0, K* k1, V* v0, V* v1, const K* src_k, const V* src_v, const K* ref, int64_t n,
           int end_bit, void* tmp, size_t tb, cudaStream_t s) {
  std::vector<float> t;
  const K* out = nullptr;
  for (int r = 0; r < 6; ++r) {
    CK(cudaMemcpyAsync(k0, src_k, sizeof(K) * n, cudaMemcpyDeviceToDevice, s));
    if (v0) CK(cudaMemcpyAsync(v0, src_v, sizeof(V) * n, cudaMemcpyDeviceToDevice, s));
    cub::DoubleBuffer<K> dk(k0, k1);
    cub::DoubleBuffer<V> dv(v0, v1);
    float ms = run<K, V, H>(dk, dv, n, end_bit, tmp, tb, s);
    if (ms < 0) return;
    if (r) t.push_back(ms);
    out = dk.Current();
  }
  std::sort(t.begin(), t.end());
  bool ok = true;
  if (ref) {
    std::vector<K> a(1 << 20), b(1 << 20);
    for (int64_t off : {int64_t(0), n / 2, n - (1 << 20)}) {
      CK(cudaMemcpy(a.data(), out + off, sizeof(K) << 20, cudaMemcpyDeviceToHost));
      CK(cudaMemcpy(b.data(), ref + off, sizeof(K) << 20, cudaMemcpyDeviceToHost));
      ok = ok && a == b;
    }
  }
  const double bytes = 2.0 * (sizeof(K) + (v0 ? sizeof(V) : 0)) * n;
  printf("%-44s median %8.3f ms  (%.2f TB/s per %d-bit pass equivalent)  %s\n", name, t[t.size() / 2],
         bytes * ((end_bit + 7) / 8) / (t[t.size() / 2] * 1e9), 8, ref ? (ok ? "same" : "DIFFERENT") : "ref");
}

int main(int argc, char** argv) {
  const int64_t n = argc > 1 ? atoll(argv[1]) : 268435456ll;
  cudaStream_t s;
  CK(cudaStreamCreate(&s));
  size_t tb = (size_t)3 << 30;
  void* tmp;
  CK(cudaMalloc(&tmp, tb));
  {  // a2 / a5: 64-bit keys, 48 significant bits
    uint64_t *src, *k0, *k1, *ref;
    CK(cudaMalloc(&src, 8 * n));
    CK(cudaMalloc(&k0, 8 * n));
    CK(cudaMalloc(&k1, 8 * n));
    CK(cudaMalloc(&ref, 8 * n));
    k_fill64<<<148 * 16, 256, 0, s>>>(src, n, 48, 1);
    using N = cub::NullType;
    N* nv = nullptr;
    bench<uint64_t, N, typename cub::detail::radix::policy_hub<uint64_t, N, OffsetT>>(
        "u64 keys 48b: default", k0, k1, nv, nv, src, nv, nullptr, n, 48, tmp, tb, s);
    {
      cub::DoubleBuffer<uint64_t> dk(k0, k1);
      cub::DoubleBuffer<N> dv(nv, nv);
      CK(cudaMemcpyAsync(k0, src, 8 * n, cudaMemcpyDeviceToDevice, s));
      run<uint64_t, N, typename cub::detail::radix::policy_hub<uint64_t, N, OffsetT>>(dk, dv, n, 48, tmp, tb, s);
      CK(cudaMemcpyAsync(ref, dk.Current(), 8 * n, cudaMemcpyDeviceToDevice, s));
    }
#define B64(OS, T, I, BITS) \
  bench<uint64_t, N, Hub<uint64_t, N, OS, T, I, BITS>>("u64 keys 48b: " #OS " " #T "x" #I " " #BITS "b", k0, k1, nv, nv, src, nv, ref, n, 48, tmp, tb, s)
    B64(true, 384, 30, 8);
    B64(true, 256, 44, 8);
    B64(true, 320, 36, 8);
    CK(cudaFree(src));
    CK(cudaFree(k0));
    CK(cudaFree(k1));
    CK(cudaFree(ref));
  }
  {  // a5 as two stable key/value sorts of 32-bit halves (rv then ru, 24 bits each) vs one 48-bit key sort
    uint32_t *ka, *kb, *va, *vb, *hi, *lo;
    CK(cudaMalloc(&ka, 4 * n));
    CK(cudaMalloc(&kb, 4 * n));
    CK(cudaMalloc(&va, 4 * n));
    CK(cudaMalloc(&vb, 4 * n));
    CK(cudaMalloc(&hi, 4 * n));
    CK(cudaMalloc(&lo, 4 * n));
    uint64_t* tmp64;
    CK(cudaMalloc(&tmp64, 8 * n));
    k_fill64<<<148 * 16, 256, 0, s>>>(tmp64, n, 48, 1);
    k_split64<<<148 * 16, 256, 0, s>>>(tmp64, n, hi, lo);
    CK(cudaFree(tmp64));
    size_t need = 0;
    cub::DoubleBuffer<uint32_t> dk(ka, kb), dv(va, vb);
    CK(cub::DeviceRadixSort::SortPairs(nullptr, need, dk, dv, n, 0, 24, s));
    std::vector<float> t;
    cudaEvent_t a, b;
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
    for (int r = 0; r < 6; ++r) {
      CK(cudaMemcpyAsync(ka, lo, 4 * n, cudaMemcpyDeviceToDevice, s));
      CK(cudaMemcpyAsync(va, hi, 4 * n, cudaMemcpyDeviceToDevice, s));
      cub::DoubleBuffer<uint32_t> k1(ka, kb), v1(va, vb);
      CK(cudaEventRecord(a, s));
      CK(cub::DeviceRadixSort::SortPairs(tmp, need, k1, v1, n, 0, 24, s));
      cub::DoubleBuffer<uint32_t> k2(v1.Current(), v1.Alternate()), v2(k1.Current(), k1.Alternate());
      CK(cub::DeviceRadixSort::SortPairs(tmp, need, k2, v2, n, 0, 24, s));
      CK(cudaEventRecord(b, s));
      CK(cudaEventSynchronize(b));
      float ms = 0;
      CK(cudaEventElapsedTime(&ms, a, b));
      if (r) t.push_back(ms);
    }
    std::sort(t.begin(), t.end());
    printf("%-44s median %8.3f ms\n", "a5 as 2 x u32/u32 pairs on 24 bits", t[t.size() / 2]);
    CK(cudaFree(ka));
    CK(cudaFree(kb));
    CK(cudaFree(va));
    CK(cudaFree(vb));
    CK(cudaFree(hi));
    CK(cudaFree(lo));
  }
  {  // a6: 32-bit key (26 bits) + 64-bit value
    uint32_t *src, *k0, *k1, *ref;
    uint64_t *vs, *v0, *v1;
    CK(cudaMalloc(&src, 4 * n));
    CK(cudaMalloc(&k0, 4 * n));
    CK(cudaMalloc(&k1, 4 * n));
    CK(cudaMalloc(&ref, 4 * n));
    CK(cudaMalloc(&vs, 8 * n));
    CK(cudaMalloc(&v0, 8 * n));
    CK(cudaMalloc(&v1, 8 * n));
    k_fill32<<<148 * 16, 256, 0, s>>>(src, vs, n, 26, 2);
    bench<uint32_t, uint64_t, typename cub::detail::radix::policy_hub<uint32_t, uint64_t, OffsetT>>(
        "u32 key 26b + u64 value: default", k0, k1, v0, v1, src, vs, nullptr, n, 26, tmp, tb, s);
    {
      cub::DoubleBuffer<uint32_t> dk(k0, k1);
      cub::DoubleBuffer<uint64_t> dv(v0, v1);
      CK(cudaMemcpyAsync(k0, src, 4 * n, cudaMemcpyDeviceToDevice, s));
      CK(cudaMemcpyAsync(v0, vs, 8 * n, cudaMemcpyDeviceToDevice, s));
      run<uint32_t, uint64_t, typename cub::detail::radix::policy_hub<uint32_t, uint64_t, OffsetT>>(dk, dv, n, 26, tmp, tb, s);
      CK(cudaMemcpyAsync(ref, dk.Current(), 4 * n, cudaMemcpyDeviceToDevice, s));
    }
#define B32(OS, T, I, BITS)                                                                                     \
  bench<uint32_t, uint64_t, Hub<uint32_t, uint64_t, OS, T, I, BITS>>("u32k+u64v 26b: " #OS " " #T "x" #I " " #BITS "b", \
                                                                     k0, k1, v0, v1, src, vs, ref, n, 26, tmp, tb, s)
    B32(true, 384, 24, 8);
    B32(true, 384, 28, 8);
    B32(true, 512, 18, 8);
    B32(true, 384, 24, 7);
    B32(true, 384, 24, 9);
    B32(false, 256, 23, 7);
  }
  return 0;
}

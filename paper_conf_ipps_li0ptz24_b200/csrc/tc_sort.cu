// tc_sort.cu — the build's large radix sorts (a2, a5, a6).
//
// A stable LSD radix sort with 8-bit digits in three launches per digit
// (reduce-then-scan, no decoupled look-back):
//   k_rs_upsweep   one CTA per 16,384-key tile: the tile's digit histogram,
//                  written digit-major (hist[d * tiles + t]);
//   DeviceScan     exclusive sum of that array = every (digit, tile)'s first
//                  output position;
//   k_rs_downsweep one CTA per tile, four sub-tiles of 4,096 keys: warp-local
//                  stable ranks by __match_any_sync, a (digit, warp) scan in
//                  shared memory, the sub-tile reordered by digit in shared
//                  memory, then written out as runs of equal digits
//                  (coalesced), each at its (digit, tile) position plus the
//                  keys of that digit in the tile's earlier sub-tiles.
// CUB's onesweep measured 2.4-2.6 ms per 8-bit pass of 268 M 64-bit keys on the
// B200 (1.65 TB/s of key traffic; profiles/r4a_c3_launches.txt); this moves
// the keys twice per pass plus one read for the histogram.
#include <cub/cub.cuh>

#include "tc_internal.cuh"

namespace tc {
namespace {

constexpr int kRsThreads = 512;
constexpr int kRsWarps = kRsThreads / 32;
constexpr int kRsItems = 8;                           // keys per thread per sub-tile
constexpr int kRsSub = kRsThreads * kRsItems;         // 4096 keys per sub-tile
constexpr int kRsSubs = 4;                            // sub-tiles per tile
constexpr int64_t kRsTile = (int64_t)kRsSub * kRsSubs;  // 16384 keys per tile
constexpr int kRsUpThreads = 256;

struct NoVal {};

template <class K>
__device__ __forceinline__ unsigned digit_of(K k, int shift, unsigned mask) {
  return (unsigned)(k >> shift) & mask;
}

// Highest lane of a peer group (its leader writes the group's count).
__device__ __forceinline__ bool is_leader(unsigned peers, int lane) {
  return (31 - __clz(peers)) == lane;
}

template <class K>
__global__ void __launch_bounds__(kRsUpThreads)
    k_rs_upsweep(const K* __restrict__ keys, int64_t n, int shift, unsigned mask, int64_t tiles,
                 uint32_t* __restrict__ hist) {
  __shared__ uint32_t wh[kRsUpThreads / 32][256];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int64_t t = blockIdx.x; t < tiles; t += gridDim.x) {
    for (int i = threadIdx.x; i < (kRsUpThreads / 32) * 256; i += kRsUpThreads) (&wh[0][0])[i] = 0;
    __syncthreads();
    const int64_t b = t * kRsTile, e = min(b + kRsTile, n);
    // a warp reads 32 consecutive keys per round (coalesced), 4 rounds in flight
    for (int64_t i0 = b + (int64_t)warp * 128; i0 < e; i0 += (int64_t)kRsUpThreads * 4) {
      K k[4];
#pragma unroll
      for (int r = 0; r < 4; ++r) {
        const int64_t i = i0 + r * 32 + lane;
        k[r] = i < e ? keys[i] : K(0);
      }
#pragma unroll
      for (int r = 0; r < 4; ++r) {
        const bool in = i0 + r * 32 + lane < e;
        const unsigned d = in ? digit_of(k[r], shift, mask) : 0xFFFFFFFFu;
        const unsigned peers = __match_any_sync(0xFFFFFFFFu, d);
        if (in && is_leader(peers, lane)) wh[warp][d] += __popc(peers);
        __syncwarp();
      }
    }
    __syncthreads();
    for (int d = threadIdx.x; d < 256; d += kRsUpThreads) {
      uint32_t s = 0;
#pragma unroll
      for (int w = 0; w < kRsUpThreads / 32; ++w) s += wh[w][d];
      if (d <= (int)mask) hist[(int64_t)d * tiles + t] = s;
    }
    __syncthreads();
  }
}

template <class K, class V, bool kVal>
struct RsSmem {
  uint32_t wh[kRsWarps][256];  // per (warp, digit): count, then the sub-tile offset
  uint32_t run[256];           // next output position of each digit for this tile
  uint32_t tot[256];           // digit count of the current sub-tile
  uint32_t start[256];         // digit start inside the sub-tile
  K sk[kRsSub];
  typename std::conditional<kVal, V, char>::type sv[kVal ? kRsSub : 1];
};

template <class K, class V, bool kVal>
__global__ void __launch_bounds__(kRsThreads, 2)
    k_rs_downsweep(const K* __restrict__ kin, K* __restrict__ kout, const V* __restrict__ vin,
                   V* __restrict__ vout, int64_t n, int shift, unsigned mask, int64_t tiles,
                   const uint32_t* __restrict__ offs) {
  extern __shared__ __align__(16) unsigned char rs_raw[];
  RsSmem<K, V, kVal>& S = *reinterpret_cast<RsSmem<K, V, kVal>*>(rs_raw);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const unsigned lt = (1u << lane) - 1u;
  for (int64_t t = blockIdx.x; t < tiles; t += gridDim.x) {
    if (threadIdx.x < 256) S.run[threadIdx.x] = threadIdx.x <= (int)mask ? offs[(int64_t)threadIdx.x * tiles + t] : 0u;
    for (int sub = 0; sub < kRsSubs; ++sub) {
      const int64_t b = t * kRsTile + (int64_t)sub * kRsSub;
      if (b >= n) break;
      const int nv = (int)(n - b < kRsSub ? n - b : kRsSub);
      // a. load: warp w owns keys [w * 256, (w + 1) * 256) of the sub-tile
      K k[kRsItems];
      V v[kVal ? kRsItems : 1];
#pragma unroll
      for (int r = 0; r < kRsItems; ++r) {
        const int i = warp * 256 + r * 32 + lane;
        k[r] = i < nv ? kin[b + i] : K(0);
        if constexpr (kVal) v[r] = i < nv ? vin[b + i] : V();
      }
      for (int i = lane; i < 256; i += 32) S.wh[warp][i] = 0;
      __syncwarp();
      // b. stable rank of each key among the warp's keys of its digit
      unsigned rk[kRsItems], dg[kRsItems];
#pragma unroll
      for (int r = 0; r < kRsItems; ++r) {
        const int i = warp * 256 + r * 32 + lane;
        // past the end: digit 255 (sorted last, never written)
        const unsigned d = i < nv ? digit_of(k[r], shift, mask) : 255u;
        const unsigned peers = __match_any_sync(0xFFFFFFFFu, d);
        const unsigned c = S.wh[warp][d];
        rk[r] = c + __popc(peers & lt);
        dg[r] = d;
        __syncwarp();
        if (is_leader(peers, lane)) S.wh[warp][d] = c + __popc(peers);
        __syncwarp();
      }
      __syncthreads();
      // c. per digit: exclusive scan over the warps, then over the digits
      if (threadIdx.x < 256) {
        const int d = threadIdx.x;
        uint32_t s = 0;
#pragma unroll
        for (int w = 0; w < kRsWarps; ++w) {
          const uint32_t c = S.wh[w][d];
          S.wh[w][d] = s;
          s += c;
        }
        S.tot[d] = s;
      }
      __syncthreads();
      if (threadIdx.x < 32) {  // one warp scans the 256 digit totals (8 per lane)
        uint32_t x[8], s = 0;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          x[j] = S.tot[lane * 8 + j];
          s += x[j];
        }
        uint32_t inc = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, inc, o);
          if (lane >= o) inc += y;
        }
        uint32_t run = inc - s;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          S.start[lane * 8 + j] = run;
          run += x[j];
        }
      }
      __syncthreads();
      // d. scatter into shared memory in (digit, warp, rank) order
#pragma unroll
      for (int r = 0; r < kRsItems; ++r) {
        const unsigned p = S.start[dg[r]] + S.wh[warp][dg[r]] + rk[r];
        S.sk[p] = k[r];
        if constexpr (kVal) S.sv[p] = v[r];
      }
      __syncthreads();
      // e. write out: consecutive positions of one digit are consecutive in
      // the output (the past-the-end keys are the sub-tile's last positions)
      for (int i = threadIdx.x; i < nv; i += kRsThreads) {
        const K x = S.sk[i];
        const unsigned d = digit_of(x, shift, mask);
        const uint32_t o = S.run[d] + (uint32_t)(i - (int)S.start[d]);
        kout[o] = x;
        if constexpr (kVal) vout[o] = S.sv[i];
      }
      __syncthreads();
      if (threadIdx.x < 256) S.run[threadIdx.x] += S.tot[threadIdx.x];
      // (the next sub-tile's first write to sk / run is behind its own barriers)
    }
    __syncthreads();
  }
}

template <class K, class V, bool kVal>
bool rs_sort(K* k0, K* k1, V* v0, V* v1, int64_t n, int begin_bit, int end_bit, cudaStream_t s) {
  const int64_t tiles = (n + kRsTile - 1) / kRsTile;
  const int passes = (end_bit - begin_bit + 7) / 8;
  DevBuf<uint32_t> hist((size_t)256 * tiles, s), offs((size_t)256 * tiles, s);
  size_t tb = 0;
  TC_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, hist.get(), offs.get(), (int64_t)256 * tiles, s));
  DevBuf<char> tmp(tb ? tb : 16, s);
  const size_t smem = sizeof(RsSmem<K, V, kVal>);
  static std::once_flag once[64];
  int dev = 0;
  TC_CUDA(cudaGetDevice(&dev));
  std::call_once(once[dev & 63], [&] {
    TC_CUDA(cudaFuncSetAttribute(k_rs_downsweep<K, V, kVal>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)smem));
  });
  int sms = 0;
  TC_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  const int grid_up = (int)std::min<int64_t>(tiles, (int64_t)sms * 8);
  const int grid_dn = (int)std::min<int64_t>(tiles, (int64_t)sms * 2);
  bool alt = false;
  for (int p = 0; p < passes; ++p) {
    const int shift = begin_bit + 8 * p;
    const int bits = std::min(8, end_bit - shift);
    const unsigned mask = (1u << bits) - 1u;
    const int64_t nd = (int64_t)(mask + 1) * tiles;
    K* ki = alt ? k1 : k0;
    K* ko = alt ? k0 : k1;
    V* vi = alt ? v1 : v0;
    V* vo = alt ? v0 : v1;
    k_rs_upsweep<K><<<grid_up, kRsUpThreads, 0, s>>>(ki, n, shift, mask, tiles, hist.get());
    TC_LAUNCH();
    TC_CUDA(cub::DeviceScan::ExclusiveSum(tmp.get(), tb, hist.get(), offs.get(), nd, s));
    k_rs_downsweep<K, V, kVal><<<grid_dn, kRsThreads, smem, s>>>(ki, ko, vi, vo, n, shift, mask, tiles,
                                                                 offs.get());
    TC_LAUNCH();
    alt = !alt;
  }
  return alt;
}

}  // namespace

bool radix_sort_keys(uint64_t* k0, uint64_t* k1, int64_t n, int begin_bit, int end_bit, cudaStream_t s) {
  NoVal* nv = nullptr;
  return rs_sort<uint64_t, NoVal, false>(k0, k1, nv, nv, n, begin_bit, end_bit, s);
}

bool radix_sort_pairs(uint32_t* k0, uint32_t* k1, uint64_t* v0, uint64_t* v1, int64_t n, int begin_bit,
                      int end_bit, cudaStream_t s) {
  return rs_sort<uint32_t, uint64_t, true>(k0, k1, v0, v1, n, begin_bit, end_bit, s);
}

}  // namespace tc

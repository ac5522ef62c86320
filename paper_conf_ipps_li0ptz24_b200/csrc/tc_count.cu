// tc_count.cu — the counting hot path: SURVEY.md §8(a) rows a7/a8/a9.
//
// What is computed (Fig. 1(b), Fig. 14): for every
// oriented edge (u,v) of the degree-ordered DAG, |N+(u) ∩ (v,∞) ∩ N+(v)|,
// the size of the intersection of u's suffix after v with v's out-list;
// their sum is T.  Edges with an empty suffix or d+(v) = 0 are skipped
// (exact, C-12); they never reach this kernel (tc_build.cu a6).
//
// How.  Live edges are grouped by their head v (the plan's
// "groups").  A CTA takes one work chunk = a run of consecutive live edges
// of near-equal cost, which covers a run of groups:
//   1. it builds, in shared memory, one open-addressing hash table per
//      group from N+(v) (the GroupTC idea of a table shared by a block of
//      edges, with TRUST-style hashing, instead of binary
//      search, which P:369/P:379 name as the cost on large graphs);
//   2. it streams the suffix keys of all its edges, flattened so that every
//      lane of every warp handles one key per step regardless of how short
//      the suffixes are (the flattened walk of P:349 / Alg. 1, with the
//      `>=` boundary test of DESIGN.md reading C-7), and probes each key in
//      its group's table;
//   3. counts go thread u32 -> warp shuffle -> CTA -> one u64 atomic.
// Tables whose N+(v) exceeds huge_degree are not staged; their keys are
// binary-searched in global memory (the TriCore-style probe).
//
// The flattened walk maps 32 consecutive flat keys to their segments with
// one coalesced load of the next 32 segment starts and a warp OR-reduce
// (__reduce_or_sync) + popc: no per-key search and no per-thread scanning.
#include <algorithm>

#include "tc_internal.cuh"

namespace tc {
namespace {

constexpr int kMaxBlock = 512;
constexpr int kUnroll = 4;  // 32-key tiles in flight per warp iteration

__device__ __forceinline__ uint32_t hash_slot(int32_t key, int lg) {
  return ((uint32_t)key * 0x9E3779B1u) >> (32 - lg);
}

// Largest s in [s_lo, s_hi) with P[s] <= k (segments are non-empty).
__device__ __forceinline__ int64_t seg_of(const int64_t* __restrict__ P, int64_t s_lo,
                                          int64_t s_hi, int64_t k) {
  int64_t lo = s_lo, hi = s_hi - 1;
  while (lo < hi) {
    int64_t mid = (lo + hi + 1) >> 1;
    if (P[mid] <= k) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// Warp-cooperative walk over the flat index range [kbeg, kend) of the
// segments [s_lo, s_hi) whose exclusive prefix is P (P[s_hi] = their end).
// Every segment must be non-empty.  load(seg, k) returns the element, then
// proc(seg, elem) consumes it; kUnroll tiles of 32 are loaded before any is
// processed so that kUnroll independent global loads are in flight per lane.
template <class Load, class Proc>
__device__ __forceinline__ void warp_walk(const int64_t* __restrict__ P, int64_t s_lo,
                                          int64_t s_hi, int64_t kbeg, int64_t kend, Load load,
                                          Proc proc) {
  if (kbeg >= kend) return;
  const int lane = threadIdx.x & 31;
  const unsigned below = (1u << lane) - 1u;
  int64_t s = seg_of(P, s_lo, s_hi, kbeg);
  for (int64_t k0 = kbeg; k0 < kend; k0 += 32 * kUnroll) {
    int64_t seg[kUnroll];
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      const int64_t t0 = k0 + 32 * u;
      const int64_t j = s + 1 + lane;
      const int64_t pos = (j <= s_hi) ? P[j] - t0 : 64;
      const unsigned bit = (pos >= 1 && pos <= 32) ? (1u << (pos - 1)) : 0u;
      const unsigned M = __reduce_or_sync(0xffffffffu, bit);
      seg[u] = s + __popc(M & below);
      s += __popc(M);
    }
    int32_t elem[kUnroll];
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      const int64_t k = k0 + 32 * u + lane;
      elem[u] = (k < kend) ? load(seg[u], k) : 0;
    }
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      const int64_t k = k0 + 32 * u + lane;
      if (k < kend) proc(seg[u], elem[u]);
    }
  }
}

__device__ __forceinline__ void hash_insert(int* __restrict__ table, int tab, int32_t key) {
  const int off = tab >> 5, lg = tab & 31;
  const uint32_t mask = (1u << lg) - 1u;
  uint32_t h = hash_slot(key, lg);
  for (;;) {
    int prev = atomicCAS(&table[off + h], -1, key);
    if (prev == -1 || prev == key) return;
    h = (h + 1) & mask;
  }
}

__device__ __forceinline__ unsigned hash_probe(const int* __restrict__ table, int tab,
                                               int32_t key) {
  const int off = tab >> 5, lg = tab & 31;
  const uint32_t mask = (1u << lg) - 1u;
  uint32_t h = hash_slot(key, lg);
  for (;;) {
    const int x = table[off + h];
    if (x == key) return 1u;
    if (x < 0) return 0u;
    h = (h + 1) & mask;
  }
}

// Binary search of key in the sorted list col[b, b+d) (huge tables only).
__device__ __forceinline__ unsigned global_probe(const int32_t* __restrict__ col, int64_t b,
                                                 int64_t d, int32_t key) {
  int64_t lo = b, hi = b + d;
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (__ldg(col + mid) < key) lo = mid + 1; else hi = mid;
  }
  return (lo < b + d && __ldg(col + lo) == key) ? 1u : 0u;
}

__global__ void __launch_bounds__(kMaxBlock)
    k_count(PlanView pv, int64_t c_begin, int64_t c_end, int64_t e_begin, int64_t e_end,
            unsigned long long* __restrict__ out) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ unsigned long long red[kMaxBlock / 32];
  const int warp = threadIdx.x >> 5, nw = blockDim.x >> 5, lane = threadIdx.x & 31;
  unsigned long long acc = 0;

  for (int64_t c = c_begin + blockIdx.x; c < c_end; c += gridDim.x) {
    const int64_t sa = max(pv.chunk_seg[c], e_begin), sb = min(pv.chunk_seg[c + 1], e_end);
    if (sa >= sb) continue;  // uniform over the CTA
    const int64_t ga = pv.seg_group[sa], gb = (int64_t)pv.seg_group[sb - 1] + 1;
    const int G = (int)(gb - ga);
    const int64_t slot0 = pv.slot_prefix[ga];
    const int nslots = (int)(pv.slot_prefix[gb] - slot0);
    int2* sInfo = reinterpret_cast<int2*>(smem);  // {tab = off << 5 | log2(slots) or -1, tmax}
    int* sHash = reinterpret_cast<int*>(sInfo + G);

    // 1. table descriptors + empty slots
    for (int i = threadIdx.x; i < G; i += blockDim.x) {
      const int64_t g = ga + i;
      const int64_t sp = pv.slot_prefix[g], ns = pv.slot_prefix[g + 1] - sp;
      const int tab = ns > 0 ? (((int)(sp - slot0)) << 5) | (31 - __clz((int)ns)) : -1;
      sInfo[i] = make_int2(tab, pv.grp_tmax[g]);
    }
    for (int i = threadIdx.x; i < nslots; i += blockDim.x) sHash[i] = -1;
    __syncthreads();

    // 2. hash N+(v) of every group touched by the chunk
    {
      const int64_t kb = pv.ins_prefix[ga], len = pv.ins_prefix[gb] - kb;
      warp_walk(
          pv.ins_prefix, ga, gb, kb + len * warp / nw, kb + len * (warp + 1) / nw,
          [&](int64_t g, int64_t k) { return __ldg(pv.col + pv.grp_ibase[g] + k); },
          [&](int64_t g, int32_t key) {
            const int tab = sInfo[g - ga].x;
            if (tab >= 0) hash_insert(sHash, tab, key);
          });
    }
    __syncthreads();

    // 3. stream the suffix keys of the chunk's edges, probe the head's table
    {
      unsigned cnt = 0;
      const int64_t kb = pv.key_prefix[sa], len = pv.key_prefix[sb] - kb;
      warp_walk(
          pv.key_prefix, sa, sb, kb + len * warp / nw, kb + len * (warp + 1) / nw,
          [&](int64_t s, int64_t k) { return __ldg(pv.col + __ldg(pv.seg_base + s) + k); },
          [&](int64_t s, int32_t key) {
            const int gl = __ldg(pv.seg_group + s) - (int)ga;
            const int2 info = sInfo[gl];
            if (key > info.y) return;  // beyond max N+(v): cannot match
            if (info.x >= 0) {
              cnt += hash_probe(sHash, info.x, key);
            } else {
              const int64_t g = ga + gl;
              const int64_t ib = pv.ins_prefix[g];
              cnt += global_probe(pv.col, pv.grp_ibase[g] + ib, pv.ins_prefix[g + 1] - ib, key);
            }
          });
      acc += cnt;
    }
    __syncthreads();  // SMEM is rebuilt by the next chunk
  }

  // 4. u64 reduction: warp shuffle -> CTA -> one atomic
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_down_sync(0xffffffffu, acc, o);
  if (lane == 0) red[warp] = acc;
  __syncthreads();
  if (warp == 0) {
    unsigned long long v = lane < nw ? red[lane] : 0ull;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
    if (lane == 0 && v) atomicAdd(out, v);
  }
}

bool g_attr_set = false;

void ensure_attr() {
  if (g_attr_set) return;
  TC_CUDA(cudaFuncSetAttribute(k_count, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               max_smem_per_block()));
  g_attr_set = true;
}

}  // namespace

int num_sms() {
  int dev = 0, v = 0;
  TC_CUDA(cudaGetDevice(&dev));
  TC_CUDA(cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev));
  return v;
}

int max_smem_per_block() {
  int dev = 0, v = 0;
  TC_CUDA(cudaGetDevice(&dev));
  TC_CUDA(cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  return v - (int)(sizeof(unsigned long long) * (kMaxBlock / 32));
}

int count_occupancy(int block, int64_t smem_bytes) {
  ensure_attr();
  int occ = 0;
  TC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_count, block, (size_t)smem_bytes));
  return occ;
}

void count_chunks(const tc_graph* g, int64_t c_begin, int64_t c_end, int64_t e_begin,
                  int64_t e_end, cudaStream_t s, unsigned long long* d_out) {
  TC_CUDA(cudaMemsetAsync(d_out, 0, sizeof(unsigned long long), s));
  const Plan& P = g->plan;
  if (c_end <= c_begin || e_end <= e_begin) return;
  ensure_attr();
  PlanView pv;
  pv.col = g->col.get();
  pv.key_prefix = P.key_prefix.get();
  pv.seg_base = P.seg_base.get();
  pv.seg_group = P.seg_group.get();
  pv.ins_prefix = P.ins_prefix.get();
  pv.grp_ibase = P.grp_ibase.get();
  pv.slot_prefix = P.slot_prefix.get();
  pv.grp_tmax = P.grp_tmax.get();
  pv.chunk_seg = P.chunk_seg.get();
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(c_end - c_begin, P.grid));
  k_count<<<grid, P.block, (size_t)P.smem_bytes, s>>>(pv, c_begin, c_end, e_begin, e_end, d_out);
  TC_LAUNCH();
}

}  // namespace tc

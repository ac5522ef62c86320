// tc_count.cu — the counting hot path: SURVEY.md §8(a) rows a7/a8/a9.
//
// What is computed (Fig. 1(b), Fig. 14): for every
// oriented edge (u,v) of the degree-ordered DAG, |N+(u) ∩ (v,∞) ∩ N+(v)|,
// the size of the intersection of u's suffix after v with v's out-list;
// their sum is T.  The plan (tc_build.cu a6) already trimmed every suffix to
// [min N+(v), max N+(v)] and dropped the edges left empty (exact, C-12).
//
// How.  Live edges are grouped by their head v.  A CTA takes
// one work chunk = a run of consecutive live edges of one class and
// near-equal cost, covering a run of groups:
//   1. it builds one hash table per group from N+(v) in shared memory (the
//      GroupTC idea of a table shared by a block of edges, with the
//      hashing TRUST uses, instead of binary search, the cost
//      P:369/P:379 name on large graphs).  Tables are two-choice (cuckoo):
//      a probe reads exactly two slots, so no warp waits on the longest of
//      32 probe chains; if an insert ever fails the chunk falls back to
//      linear probing;
//   2. it streams the edges' suffix keys and probes the head's table:
//      LONG class (suffix >= long_min keys): one warp walks one edge in
//        32-key tiles, coalesced, with warp-uniform bookkeeping;
//      SHORT class: the keys of all the chunk's edges are flattened over the
//        lanes (the flattened walk of P:349 / Alg. 1 with the `>=` boundary
//        of DESIGN.md reading C-7), 32 consecutive keys mapped to their
//        edges with one SMEM load, a warp OR-reduce and popc;
//      (degree-bucketed dispatch, the TRUST/Fox idea of P:176/P:254);
//   3. counts go thread u32 -> warp shuffle -> CTA -> one u64 atomic.
// Tables whose N+(v) exceeds huge_degree are not staged; their keys are
// binary-searched in global memory (the TriCore-style probe).
#include <algorithm>

#include "tc_internal.cuh"

namespace tc {
namespace {

constexpr int kMaxBlock = 512;
constexpr int kUnroll = 4;     // tiles in flight per warp iteration
constexpr int kMaxKicks = 96;  // cuckoo displacement bound before the linear fallback

// Table descriptor tab = (slot offset << 5) | sh with sh = 32 - log2(slots):
// the slot of a key is the top log2(slots) bits of a multiplicative hash.
__device__ __forceinline__ uint32_t hash1(int32_t key, int sh) {
  return ((uint32_t)key * 0x9E3779B1u) >> sh;
}
__device__ __forceinline__ uint32_t hash2(int32_t key, int sh) {
  return ((uint32_t)key * 0x85EBCA77u + 0x7F4A7C15u) >> sh;
}

// Largest s in [s_lo, s_hi) with P[s] <= k (segments are non-empty).
template <class T>
__device__ __forceinline__ T seg_of(const T* __restrict__ P, T s_lo, T s_hi, T k) {
  T lo = s_lo, hi = s_hi - 1;
  while (lo < hi) {
    T mid = (lo + hi + 1) >> 1;
    if (P[mid] <= k) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// Warp walk over the flat range [kbeg, kend) of the segments [s_lo, s_hi)
// with (global, int64) exclusive prefix P; used to insert N+(v) keys.
template <class Proc>
__device__ __forceinline__ void warp_walk_global(const int64_t* __restrict__ P, int64_t s_lo,
                                                 int64_t s_hi, int64_t kbeg, int64_t kend,
                                                 const int32_t* __restrict__ col,
                                                 const int64_t* __restrict__ base, Proc proc) {
  if (kbeg >= kend) return;
  const int lane = threadIdx.x & 31;
  const unsigned below = (1u << lane) - 1u;
  int64_t s = seg_of<int64_t>(P, s_lo, s_hi, kbeg);
  for (int64_t k0 = kbeg; k0 < kend; k0 += 32) {
    const int64_t j = s + 1 + lane;
    const int64_t pos = (j <= s_hi) ? P[j] - k0 : 64;
    const unsigned bit = (pos >= 1 && pos <= 32) ? (1u << (pos - 1)) : 0u;
    const unsigned M = __reduce_or_sync(0xffffffffu, bit);
    const int64_t seg = s + __popc(M & below);
    s += __popc(M);
    const int64_t k = k0 + lane;
    if (k < kend) proc(seg, __ldg(col + __ldg(base + seg) + k));
  }
}

__device__ __forceinline__ bool cuckoo_insert(int* __restrict__ T, int tab, int32_t key) {
  const int off = tab >> 5, sh = tab & 31;
  uint32_t pos = hash1(key, sh);
  for (int i = 0; i < kMaxKicks; ++i) {
    const int old = atomicExch(&T[off + pos], key);
    if (old < 0) return true;
    key = old;  // displaced: move it to its other slot
    const uint32_t p1 = hash1(key, sh);
    pos = (pos == p1) ? hash2(key, sh) : p1;
  }
  return false;  // `key` is homeless: the chunk rebuilds with linear probing
}

__device__ __forceinline__ void linear_insert(int* __restrict__ T, int tab, int32_t key) {
  const int off = tab >> 5, sh = tab & 31;
  const uint32_t mask = 0xffffffffu >> sh;
  uint32_t h = hash1(key, sh);
  for (;;) {
    const int prev = atomicCAS(&T[off + h], -1, key);
    if (prev == -1 || prev == key) return;
    h = (h + 1) & mask;
  }
}

// Binary search of key in the sorted list col[b, b+d) (huge tables only).
__device__ __noinline__ unsigned global_probe(const int32_t* __restrict__ col, int64_t b, int64_t d,
                                              int32_t key) {
  int64_t lo = b, hi = b + d;
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (__ldg(col + mid) < key) lo = mid + 1; else hi = mid;
  }
  return (lo < b + d && __ldg(col + lo) == key) ? 1u : 0u;
}

// Membership of key in one SMEM table: T = first slot, sh = 32 - log2(slots).
// Keys are >= 0, empty slots hold -1, and the sentinel -2 (padding lanes)
// never matches and always terminates.
template <bool kLinear>
__device__ __forceinline__ unsigned table_probe(const int* __restrict__ T, int sh, int32_t key) {
  if (!kLinear) {
    // two-choice table: a key lives at hash1 or hash2; both reads are issued
    const int x1 = T[hash1(key, sh)];
    const int x2 = T[hash2(key, sh)];
    return (x1 == key) | (x2 == key);
  }
  const uint32_t mask = 0xffffffffu >> sh;
  uint32_t h = hash1(key, sh);
  for (;;) {
    const int x = T[h];
    if (x == key) return 1u;
    if (x < 0) return 0u;
    h = (h + 1) & mask;
  }
}

// Membership through a descriptor (tab = off << 5 | sh, or -1 = huge table
// of group g, probed by binary search in global memory).
template <bool kLinear, bool kHuge>
__device__ __forceinline__ unsigned probe(const int* __restrict__ H, int tab, int32_t key,
                                          const PlanView& pv, int64_t g) {
  if (kHuge && tab < 0) {
    const int64_t ib = pv.ins_prefix[g];
    return global_probe(pv.col, pv.grp_ibase[g] + ib, pv.ins_prefix[g + 1] - ib, key);
  }
  return table_probe<kLinear>(H + (tab >> 5), tab & 31, key);
}

struct ChunkSmem {
  int64_t* sB;  // long: key start in col; short: start - (chunk-relative first key)
  int* sA;      // [S+1] long: tile prefix; short: key prefix (chunk-relative)
  int* sC;      // long: suffix length
  int* sD;      // group index (chunk-local)
  int* sInfo;   // [G] table descriptor
  int* sHash;   // slots
};

// LONG class: the warp owns tiles [t0, t1) of the chunk; each tile is 32
// consecutive keys of one edge.  The warp walks edge by edge (warp-uniform
// bookkeeping); inside an edge, lane l reads keys l, l+32, ... through one
// pointer with immediate offsets, kUnroll tiles in flight; lanes past the
// end carry the never-matching sentinel so the probes run unpredicated.
template <bool kLinear, bool kHuge>
__device__ __forceinline__ unsigned walk_long(const ChunkSmem& c, int S, int t0, int t1,
                                              const PlanView& pv, int64_t ga) {
  unsigned cnt = 0;
  if (t0 >= t1) return cnt;
  const int lane = threadIdx.x & 31;
  int s = seg_of<int>(c.sA, 0, S, t0);
  for (int t = t0; t < t1; ++s) {
    const int ts = c.sA[s], te = min(c.sA[s + 1], t1);
    const int done = (t - ts) << 5;                             // keys of this edge before tile t
    const int lim = min(c.sC[s] - done, (te - t) << 5) - lane;  // lane's keys: 32*i < lim
    const int32_t* __restrict__ p = pv.col + c.sB[s] + done + lane;
    const int gl = c.sD[s];
    const int tab = c.sInfo[gl];
    t = te;
    if (kHuge && tab < 0) {
      for (int i = 0; i < lim; i += 32) cnt += probe<kLinear, true>(c.sHash, tab, __ldg(p + i), pv, ga + gl);
      continue;
    }
    const int* __restrict__ T = c.sHash + (tab >> 5);
    const int sh = tab & 31;
    for (int i = 0; i < lim; i += 32 * kUnroll) {
      int32_t key[kUnroll];
#pragma unroll
      for (int u = 0; u < kUnroll; ++u) key[u] = (i + 32 * u < lim) ? __ldg(p + i + 32 * u) : -2;
#pragma unroll
      for (int u = 0; u < kUnroll; ++u) cnt += table_probe<kLinear>(T, sh, key[u]);
    }
  }
  return cnt;
}

// SHORT class: the warp owns the flat keys [k0w, k1w) of the chunk.
template <bool kLinear, bool kHuge>
__device__ __forceinline__ unsigned walk_short(const ChunkSmem& c, int S, int k0w, int k1w,
                                               const PlanView& pv, int64_t ga) {
  unsigned cnt = 0;
  if (k0w >= k1w) return cnt;
  const int lane = threadIdx.x & 31;
  const unsigned below = (1u << lane) - 1u;
  int s = seg_of<int>(c.sA, 0, S, k0w);
  for (int k0 = k0w; k0 < k1w; k0 += 32 * kUnroll) {
    int seg[kUnroll];
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      const int t0 = k0 + 32 * u;
      const int j = s + 1 + lane;
      const int pos = (j <= S) ? c.sA[j] - t0 : 64;
      const unsigned bit = (pos >= 1 && pos <= 32) ? (1u << (pos - 1)) : 0u;
      const unsigned M = __reduce_or_sync(0xffffffffu, bit);
      seg[u] = s + __popc(M & below);
      s += __popc(M);
    }
    int32_t key[kUnroll];
    int gl[kUnroll];
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      const int k = k0 + 32 * u + lane;
      key[u] = 0;
      gl[u] = 0;
      if (k < k1w) {
        key[u] = __ldg(pv.col + c.sB[seg[u]] + k);
        gl[u] = c.sD[seg[u]];
      }
    }
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      const int k = k0 + 32 * u + lane;
      if (k < k1w) cnt += probe<kLinear, kHuge>(c.sHash, c.sInfo[gl[u]], key[u], pv, ga + gl[u]);
    }
  }
  return cnt;
}

__global__ void __launch_bounds__(kMaxBlock, 3)  // 3 CTAs x 16 warps per SM
    k_count(PlanView pv, int64_t c_begin, int64_t c_end, int64_t e_begin, int64_t e_end,
            unsigned long long* __restrict__ out) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ unsigned long long red[kMaxBlock / 32];
  __shared__ int sFail;
  const int warp = threadIdx.x >> 5, nw = blockDim.x >> 5, lane = threadIdx.x & 31;
  unsigned long long acc = 0;

  for (int64_t cix = c_begin + blockIdx.x; cix < c_end; cix += gridDim.x) {
    const int64_t sa = max(pv.chunk_seg[cix], e_begin), sb = min(pv.chunk_seg[cix + 1], e_end);
    if (sa >= sb) continue;  // uniform over the CTA
    const bool is_long = cix < pv.n_long_chunks;
    const int S = (int)(sb - sa);
    const int64_t ga = pv.seg_group[sa], gb = (int64_t)pv.seg_group[sb - 1] + 1;
    const int G = (int)(gb - ga);
    const int64_t slot0 = pv.slot_prefix[ga];
    const int nslots = (int)(pv.slot_prefix[gb] - slot0);
    ChunkSmem c;
    c.sB = reinterpret_cast<int64_t*>(smem);
    c.sA = reinterpret_cast<int*>(c.sB + S);
    c.sC = c.sA + S + 1;
    c.sD = c.sC + S;
    c.sInfo = c.sD + S;
    // 16-B aligned start of the slots, as an int offset from the (aligned) base
    // so the compiler keeps every table access in the shared window (LDS/ATOMS)
    c.sHash = reinterpret_cast<int*>(smem) + ((2 * S + (S + 1) + S + S + G + 3) & ~3);

    // 1. stage the chunk's edges and table descriptors; empty slots
    const int64_t kp0 = pv.key_prefix[sa];
    for (int i = threadIdx.x; i <= S; i += blockDim.x) {
      const int64_t sg = sa + i;
      const int rel = (int)(pv.key_prefix[sg] - kp0);
      c.sA[i] = is_long ? (rel >> 5) : rel;
      if (i < S) {
        c.sB[i] = is_long ? pv.seg_start[sg] : pv.seg_start[sg] - rel;
        c.sC[i] = pv.seg_len[sg];
        c.sD[i] = pv.seg_group[sg] - (int)ga;
      }
    }
    int huge = 0;
    for (int i = threadIdx.x; i < G; i += blockDim.x) {
      const int64_t sp = pv.slot_prefix[ga + i], ns = pv.slot_prefix[ga + i + 1] - sp;
      c.sInfo[i] = ns > 0 ? (((int)(sp - slot0)) << 5) | (32 - (31 - __clz((int)ns))) : -1;
      huge |= ns == 0;
    }
    {
      int4* h4 = reinterpret_cast<int4*>(c.sHash);
      for (int i = threadIdx.x; i < (nslots >> 2); i += blockDim.x) h4[i] = make_int4(-1, -1, -1, -1);
      for (int i = (nslots & ~3) + threadIdx.x; i < nslots; i += blockDim.x) c.sHash[i] = -1;
    }
    if (threadIdx.x == 0) sFail = 0;
    const bool any_huge = __syncthreads_or(huge);

    // 2. hash N+(v) of every group touched by the chunk
    bool linear = pv.probe_mode == 1;
    const int64_t ib = pv.ins_prefix[ga], ilen = pv.ins_prefix[gb] - ib;
    const int64_t iw0 = ib + ilen * warp / nw, iw1 = ib + ilen * (warp + 1) / nw;
    if (linear) {
      warp_walk_global(pv.ins_prefix, ga, gb, iw0, iw1, pv.col, pv.grp_ibase,
                       [&](int64_t g, int32_t key) {
                         const int tab = c.sInfo[g - ga];
                         if (tab >= 0) linear_insert(c.sHash, tab, key);
                       });
    } else {
      bool ok = true;
      warp_walk_global(pv.ins_prefix, ga, gb, iw0, iw1, pv.col, pv.grp_ibase,
                       [&](int64_t g, int32_t key) {
                         const int tab = c.sInfo[g - ga];
                         if (tab >= 0 && !cuckoo_insert(c.sHash, tab, key)) ok = false;
                       });
      if (!ok) sFail = 1;
    }
    __syncthreads();
    if (!linear && sFail) {  // uniform: rebuild this chunk's tables with linear probing
      linear = true;
      for (int i = threadIdx.x; i < nslots; i += blockDim.x) c.sHash[i] = -1;
      __syncthreads();  // (rare path: scalar init is fine)
      warp_walk_global(pv.ins_prefix, ga, gb, iw0, iw1, pv.col, pv.grp_ibase,
                       [&](int64_t g, int32_t key) {
                         const int tab = c.sInfo[g - ga];
                         if (tab >= 0) linear_insert(c.sHash, tab, key);
                       });
      __syncthreads();
    }

    // 3. stream the chunk's suffix keys and probe the heads' tables
    const int NU = c.sA[S];
    const int w0 = (int)((int64_t)NU * warp / nw), w1 = (int)((int64_t)NU * (warp + 1) / nw);
    unsigned cnt;
    if (is_long) {
      if (any_huge)
        cnt = linear ? walk_long<true, true>(c, S, w0, w1, pv, ga) : walk_long<false, true>(c, S, w0, w1, pv, ga);
      else
        cnt = linear ? walk_long<true, false>(c, S, w0, w1, pv, ga) : walk_long<false, false>(c, S, w0, w1, pv, ga);
    } else {
      if (any_huge)
        cnt = linear ? walk_short<true, true>(c, S, w0, w1, pv, ga) : walk_short<false, true>(c, S, w0, w1, pv, ga);
      else
        cnt = linear ? walk_short<true, false>(c, S, w0, w1, pv, ga) : walk_short<false, false>(c, S, w0, w1, pv, ga);
    }
    acc += cnt;
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
  cudaFuncAttributes fa;
  TC_CUDA(cudaFuncGetAttributes(&fa, k_count));
  return v - (int)fa.sharedSizeBytes;  // dynamic + static must fit the opt-in limit
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
  pv.seg_start = P.seg_start.get();
  pv.seg_len = P.seg_len.get();
  pv.seg_group = P.seg_group.get();
  pv.ins_prefix = P.ins_prefix.get();
  pv.grp_ibase = P.grp_ibase.get();
  pv.slot_prefix = P.slot_prefix.get();
  pv.chunk_seg = P.chunk_seg.get();
  pv.n_long_chunks = P.n_long_chunks;
  pv.probe_mode = P.opt.probe_mode;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(c_end - c_begin, P.grid));
  k_count<<<grid, P.block, (size_t)P.smem_bytes, s>>>(pv, c_begin, c_end, e_begin, e_end, d_out);
  TC_LAUNCH();
}

}  // namespace tc

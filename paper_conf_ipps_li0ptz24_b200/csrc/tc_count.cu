// tc_count.cu — the counting hot path: SURVEY.md §8(a) rows a7/a8/a9.
//
// What is computed (Fig. 1(b), Fig. 14): for every
// oriented edge (u,v) of the degree-ordered DAG, |N+(u) ∩ (v,∞) ∩ N+(v)|,
// the size of the intersection of u's suffix after v with v's out-list;
// their sum is T.  The plan (tc_build.cu a6) already trimmed every suffix to
// [min N+(v), max N+(v)] and dropped the edges left empty (exact, C-12/C-21).
//
// How.  Live edges are grouped by their head v.  Work comes
// in chunks = runs of consecutive live edges of one class and near-equal
// cost, covering a run of groups.  Two kernels, one per class:
//   k_count (LONG class, suffix >= long_min keys): one persistent 1024-thread
//   CTA per SM, warp-specialised, with three chunk slots in shared memory.
//   PRODUCER warps (1/4 of the CTA, in two groups that fill alternate
//     chunks concurrently) stage the CTA's next chunks into free
//     slots: each chunk's edges, its per-32-key tile descriptors, and one table per
//     group built from N+(v) (the GroupTC idea of a table shared by a block
//     of edges): a bitmap of N+(v)'s rank window (one probe per key)
//     or a two-choice (cuckoo) hash, as in TRUST, instead of the
//     binary search P:369/P:379 name as the cost on large graphs; a failed
//     cuckoo insert rebuilds the chunk's tables with linear probing.  They
//     hand the slot over with an mbarrier.
//   CONSUMER warps walk the chunk's tiles (32 consecutive keys of one edge,
//     coalesced, 8 tiles per batch in flight per lane), probe the heads'
//     tables and release the slot with an mbarrier.
//   k_count_flat (SHORT class): 4 CTAs x 384 threads per SM, every warp
//     stages, builds and probes one chunk per CTA; the keys of all the chunk's
//     edges are flattened over the lanes (the flattened walk of P:349 / Alg. 1
//     with the `>=` boundary of DESIGN.md reading C-7), 32 consecutive keys
//     mapped to their edges with one SMEM load, a warp OR-reduce and popc
//     (degree-bucketed dispatch, the TRUST/Fox idea of P:176/P:254).
//   Counts go thread u32 -> u64 -> warp shuffle -> CTA -> one atomic;
//   with the fused cross-GPU sum (f4) the last CTA of the last launch adds the
//   partial into every rank's symmetric buffer (tc_fused.cuh).
// Tables whose N+(v) exceeds huge_degree are not staged; their keys are
// binary-searched in global memory (the TriCore-style probe).
#include <algorithm>
#include <cstring>
#include <mutex>

#include "tc_internal.cuh"

namespace tc {
namespace {

constexpr int kMaxBlock = 1024;  // warp-specialised kernel (long class)
#ifndef TC_FLAT_BLOCK
#define TC_FLAT_BLOCK 384
#endif
#ifndef TC_FLAT_CTAS
#define TC_FLAT_CTAS 4
#endif
constexpr int kFlatBlock = TC_FLAT_BLOCK;  // flat kernel (short class) ...
constexpr int kFlatCTAs = TC_FLAT_CTAS;    // ... and its CTAs per SM
constexpr int kUnrollLong = 8;   // tail batch of the long class
#ifndef TC_BATCH_LONG
#define TC_BATCH_LONG 8
#endif
constexpr int kBatchLong = TC_BATCH_LONG;  // tiles per batch: key loads in flight per lane
#ifndef TC_PF_SHORT
#define TC_PF_SHORT 1  // produce: L2 prefetch of every short-class edge's keys at staging (r2y: C2 -1.6%)
#endif
#ifndef TC_L2PF
#define TC_L2PF 1  // walk_long: L2 prefetch of the key lines TC_L2PF batches ahead (0: off;
#endif             // r2v C3 k_count 42.2 -> 38.9 ms, C4 564 -> 545 ms with 1)
#ifndef TC_UNROLL_SHORT
#define TC_UNROLL_SHORT 2
#endif
constexpr int kUnrollShort = TC_UNROLL_SHORT;  // tiles in flight per consumer warp (short class)
constexpr int kMaxKicks = 96;    // cuckoo displacement bound before the linear fallback (Tuning::max_kicks)
constexpr int kMaxSlots = 4;     // chunk slots in SMEM (runtime count: Tuning::slots)

// ------------------------------------------------------------------ mbarrier (PTX)
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.shared::cta.b64 st, [%0];\n\t}" ::"r"(smem_u32(b))
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity, uint32_t hint_ns) {
  if (hint_ns) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tWAITH_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n\t"
        "@!p bra WAITH_%=;\n\t}" ::"r"(smem_u32(b)),
        "r"(parity), "r"(hint_ns)
        : "memory");
  } else {
    asm volatile(
        "{\n\t.reg .pred p;\n\tWAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(b)),
        "r"(parity)
        : "memory");
  }
}
// The two waits of the count kernel as separate functions, so profiles
// attribute consumer (slot full) and producer (slot empty) waiting apart.
__device__ __noinline__ void wait_full(uint64_t* b, uint32_t parity, uint32_t hint_ns) {
  mbar_wait(b, parity, hint_ns);
}
__device__ __noinline__ void wait_empty(uint64_t* b, uint32_t parity, uint32_t hint_ns) {
  mbar_wait(b, parity, hint_ns);
}
__device__ __forceinline__ void named_sync(int id, int nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
// Named barrier that also ORs a predicate over its participants.
__device__ __forceinline__ int named_sync_or(int id, int nthreads, int pred) {
  int r;
  asm volatile(
      "{\n\t.reg .pred p, q;\n\tsetp.ne.s32 p, %1, 0;\n\t"
      "bar.red.or.pred q, %2, %3, p;\n\tselp.s32 %0, 1, 0, q;\n\t}"
      : "=r"(r)
      : "r"(pred), "r"(id), "r"(nthreads)
      : "memory");
  return r;
}

// Diagnostic counters (tc_counters): [0] chunks whose two-choice table
// inserts failed and were rebuilt with linear probing.  Touched only on that
// rare path.
__device__ unsigned long long g_counters[4];

// ------------------------------------------------------------------ hashing
// A table is (off, n): n slots starting at sHash[off].  The slot of a key is
// a multiplicative hash mapped onto [0, n) by a 32x32 -> high-32 multiply
// (no power-of-two rounding, so the load stays at 1/table_factor).
__device__ __forceinline__ uint32_t hash1(int32_t key, uint32_t n) {
  return __umulhi((uint32_t)key * 0x9E3779B1u, n);
}
__device__ __forceinline__ uint32_t hash2(int32_t key, uint32_t n) {
  return __umulhi((uint32_t)key * 0x85EBCA77u + 0x7F4A7C15u, n);
}

__device__ __forceinline__ bool cuckoo_insert(int* __restrict__ T, uint32_t n, int32_t key,
                                              int max_kicks) {
  uint32_t pos = hash1(key, n);
  for (int i = 0; i < max_kicks; ++i) {
    const int old = atomicExch(&T[pos], key);
    if (old < 0) return true;
    key = old;  // displaced: move it to its other slot
    const uint32_t p1 = hash1(key, n);
    pos = (pos == p1) ? hash2(key, n) : p1;
  }
  return false;  // `key` is homeless: the chunk rebuilds with linear probing
}

__device__ __forceinline__ void linear_insert(int* __restrict__ T, uint32_t n, int32_t key) {
  uint32_t h = hash1(key, n);
  for (;;) {
    const int prev = atomicCAS(&T[h], -1, key);
    if (prev == -1 || prev == key) return;
    h = (h + 1 == n) ? 0 : h + 1;
  }
}

// Support mode (8-B entries {key, payload}; empty = all ones).  The same
// two-choice / linear schemes, moving the payload with its key.
__device__ __forceinline__ bool cuckoo_insert64(unsigned long long* __restrict__ T, uint32_t n,
                                                int32_t key, unsigned long long e, int max_kicks) {
  uint32_t pos = hash1(key, n);
  for (int i = 0; i < max_kicks; ++i) {
    const unsigned long long old = atomicExch(&T[pos], e);
    if ((int)(uint32_t)old < 0) return true;
    e = old;
    key = (int)(uint32_t)old;
    const uint32_t p1 = hash1(key, n);
    pos = (pos == p1) ? hash2(key, n) : p1;
  }
  return false;
}

__device__ __forceinline__ void linear_insert64(unsigned long long* __restrict__ T, uint32_t n,
                                                int32_t key, unsigned long long e) {
  uint32_t h = hash1(key, n);
  for (;;) {
    const unsigned long long prev = atomicCAS(&T[h], ~0ull, e);
    if (prev == ~0ull || (int)(uint32_t)prev == key) return;
    h = (h + 1 == n) ? 0 : h + 1;
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

// Membership of key in the SMEM table T[0, n).  Keys are >= 0, empty slots
// hold -1, and the sentinel -2 (padding lanes) never matches and always
// terminates (a table has more slots than keys).
template <bool kLinear>
__device__ __forceinline__ unsigned table_probe(const int* __restrict__ T, uint32_t n, int32_t key) {
  if (!kLinear) {
    // two-choice table: a key lives at hash1 or hash2; both reads are issued
    // unconditionally (a read of hash2 that waits on hash1 measured slower)
    const int x1 = T[hash1(key, n)];
    const int x2 = T[hash2(key, n)];
    return (unsigned)(x1 == key) | (unsigned)(x2 == key);
  }
  uint32_t h = hash1(key, n);
  for (;;) {
    const int x = T[h];
    if (x == key) return 1u;
    if (x < 0) return 0u;
    h = (h + 1 == n) ? 0 : h + 1;
  }
}

// Membership in a table of either kind: T = its first word, code = n >= 2
// (hash, n slots) or -(first rank word) <= 0 (bitmap of the rank window,
// bits inverted so that an initialised word is all ones).  Padding lanes
// (key < 0) never match and read only inside the table.
template <bool kLinear>
__device__ __forceinline__ unsigned any_probe(const int* __restrict__ T, int code, int32_t key) {
  if (code <= 0) {
    const int w = max((key >> 5) + code, 0);
    return (((~(unsigned)T[w]) >> (key & 31)) & 1u) & (unsigned)(key >= 0);
  }
  return table_probe<kLinear>(T, (uint32_t)code, key);
}

__device__ __forceinline__ void bitmap_insert(int* __restrict__ T, int code, int32_t key) {
  atomicAnd(&T[(key >> 5) + code], ~(1 << (key & 31)));
}

__device__ __forceinline__ unsigned huge_probe(const PlanView& pv, int64_t g, int32_t key) {
  const int64_t ib = pv.ins_prefix[g];
  return global_probe(pv.col, pv.grp_ibase[g] + ib, pv.ins_prefix[g + 1] - ib, key);
}

// ------------------------------------------------------------------ chunk slot
// One slot = the staged edges, groups, tiles and tables of one chunk; layout
// in chunk_smem_bytes (tc_internal.cuh).
struct SlotHdr {
  long long sa, ga;
  int S, G, T, nslots, is_long, linear, done, huge, next, pad;  // next: work-grab counter
};

struct ChunkSmem {
  // long class: one descriptor per 32-key tile as four int arrays of T4 =
  // round4(T) entries (structure of arrays: one LDS.128 reads a field of 4
  // tiles).  Count mode: sT0 = col index of the tile's first key, sT1 =
  // valid lanes, sT2/sT3 = table (walk_long); support mode: key position
  // lo/hi, chunk-local edge, valid lanes (walk_long_sup).
  int *sT0, *sT1, *sT2, *sT3;
  int64_t* sB;   // long: key start in col; short: start - (chunk-relative first key)
  int64_t* sGB;  // group: row start of N+(v) - sGP (so col[sGB[g] + k] is insert k)
  int2* sInfo;   // [G] table {word offset, code}; offset -1 = huge
  int* sA;       // [S+1] long: tile prefix; short: key prefix (chunk-relative)
  int* sC;       // suffix length
  int* sD;       // group index (chunk-local)
  int* sGP;      // [G+1] insert prefix (chunk-relative)
  int* sHash;    // slots (support mode: 8-B entries, see produce)
  int64_t* sE;   // support mode only: [S] CSR position of each edge (u,v)
};

__device__ __forceinline__ ChunkSmem slot_view(unsigned char* region, int S, int G, int T) {
  ChunkSmem c;
  const int T4 = (T + 3) & ~3;
  c.sT0 = reinterpret_cast<int*>(region);
  c.sT1 = c.sT0 + T4;
  c.sT2 = c.sT1 + T4;
  c.sT3 = c.sT2 + T4;
  c.sB = reinterpret_cast<int64_t*>(c.sT3 + T4);
  c.sGB = c.sB + S;
  c.sInfo = reinterpret_cast<int2*>(c.sGB + G);
  c.sA = reinterpret_cast<int*>(c.sInfo + G);
  c.sC = c.sA + S + 1;
  c.sD = c.sC + S;
  c.sGP = c.sD + S;
  // 16-B aligned start of the slots as an int offset from the aligned region
  // base, so every table access stays in the shared window (LDS/ATOMS)
  c.sHash = reinterpret_cast<int*>(region) +
            ((4 * T4 + 2 * S + 2 * G + 2 * G + (S + 1) + 2 * S + (G + 1) + 3) & ~3);
  c.sE = nullptr;
  return c;
}

// Support mode (f1): every table entry is 8 B (a hash slot {key, index in
// N+(v)}, a bitmap word {bits, members in earlier words}), followed by the
// edges' own CSR positions.  Bytes: chunk_smem_bytes + 4*slots + 8*S.
__device__ __forceinline__ ChunkSmem slot_view_sup(unsigned char* region, int S, int G, int T,
                                                   int nslots) {
  ChunkSmem c = slot_view(region, S, G, T);
  c.sE = reinterpret_cast<int64_t*>(c.sHash + 2 * nslots);
  return c;
}

// Largest s in [0, S) with P[s] <= k (segments are non-empty).
__device__ __forceinline__ int seg_of(const int* __restrict__ P, int S, int k) {
  int lo = 0, hi = S - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (P[mid] <= k) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// Warp walk over the flat range [kbeg, kend) of the segments [0, S) whose
// exclusive prefix is the SMEM array P (P[S] = their end; segments non-empty).
// 32 consecutive flat indices are mapped to their segments with one SMEM
// load of the next 32 starts, a warp OR-reduce of a position mask and popc.
// kU tiles are mapped, then load(seg, k) is issued for all of them (kU
// independent global loads in flight per lane), then proc(seg, k, value).
template <int kU, class Load, class Proc>
__device__ __forceinline__ void warp_walk(const int* __restrict__ P, int S, int kbeg, int kend,
                                          Load load, Proc proc) {
  if (kbeg >= kend) return;
  const int lane = threadIdx.x & 31;
  const unsigned below = (1u << lane) - 1u;
  int s = seg_of(P, S, kbeg);
  for (int k0 = kbeg; k0 < kend; k0 += 32 * kU) {
    int seg[kU];
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const int t0 = k0 + 32 * u;
      const int j = s + 1 + lane;
      const int pos = (j <= S) ? P[j] - t0 : 64;
      const unsigned bit = (pos >= 1 && pos <= 32) ? (1u << (pos - 1)) : 0u;
      const unsigned M = __reduce_or_sync(0xffffffffu, bit);
      seg[u] = s + __popc(M & below);
      s += __popc(M);
    }
    int32_t val[kU];
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const int k = k0 + 32 * u + lane;
      val[u] = k < kend ? load(seg[u], k) : 0;
    }
#pragma unroll
    for (int u = 0; u < kU; ++u)
      if (k0 + 32 * u + lane < kend) proc(seg[u], k0 + 32 * u + lane, val[u]);
  }
}

// ------------------------------------------------------------------ consumers
// LONG class: the warp owns tiles [t0, t1) of the chunk.  Each tile is 32
// consecutive keys of one edge, described by one 16-B sTile entry the
// producers wrote: {x = col index of the tile's first key (m < 2^32),
// y = valid lanes (1..32), z/w = its table: w = 0 bitmap whose word for key k
// is sHash[(k >> 5) + z]; w >= 2 hash of w slots at sHash[z]; w = -1 huge,
// z = -1 - (chunk-local group)}.  kUnrollLong tiles are loaded per step
// (kUnrollLong key loads in flight per lane across edge boundaries, no
// per-edge bookkeeping).  Padding lanes re-load the tile's last valid key
// (always a legal address and a legal table read) and their hit is masked,
// so every lane probes unpredicated.
// zw = (code << 6) | first valid lane (see produce): code 0 bitmap, >= 2 hash
// slots, -1 huge; first valid lane 32 = none.
// Returns the lane's hit WITHOUT the valid-lane mask (the caller adds it
// under `lane >= first valid lane`: one ISETP + a predicated IADD).
template <bool kLinear, bool kHuge>
__device__ __forceinline__ unsigned probe_tile(const ChunkSmem& c, int z, int zw, int32_t key,
                                               int lane, const PlanView& pv, int64_t ga) {
  // z of a staged table is relative to the slot base c.sT0 (the producer
  // added the table area's offset), so an address is ((key >> 5) + z) * 4 +
  // slot base
  const int w = zw >> 6;
  if (w == 0) {
    const unsigned word = (unsigned)c.sT0[(key >> 5) + z];
    return (__funnelshift_r(word, 0u, (unsigned)key) & 1u) ^ 1u;  // bit key & 31 of ~word
  }
  if (!kHuge || w > 0) return table_probe<kLinear>(c.sT0 + z, (uint32_t)w, key);
  return lane >= (zw & 63) ? huge_probe(pv, ga + (-1 - z), key) : 0u;
}

// Tiles [t0, t1), t0 a multiple of 8 (the consumer split keeps it so): each
// descriptor field of an 8-tile batch is two aligned LDS.128.  Every lane of a
// tile loads a key of the tile's own edge (x + lane; a partial last tile was
// shifted back and its first lanes are masked), so a key address needs only
// the x field.  (Software-pipelining batch b+1's loads under batch b's probes
// measured slower: 4-tile batches 66 ms, 8-tile batches spill, vs 62.5 ms.)
template <int kB>
__device__ __forceinline__ void load_batch(const ChunkSmem& c, const int32_t* colL, int t,
                                           int32_t (&key)[kB]) {
  int x[kB];
#pragma unroll
  for (int q = 0; q < kB; q += 4)
    *reinterpret_cast<int4*>(x + q) = *reinterpret_cast<const int4*>(c.sT0 + t + q);
  // colL = col + lane, opaque to the compiler (lane_base): each key address is
  // ONE IMAD.WIDE.U32 x * 4 + colL (left to itself, nvcc re-associates it into
  // a 64-bit add-with-carry + LEA pair, 4 instructions per key)
#pragma unroll
  for (int u = 0; u < kB; ++u) key[u] = __ldg(colL + (uint32_t)x[u]);
}

// col + lane in a register the compiler cannot see through.
__device__ __forceinline__ const int32_t* lane_base(const int32_t* col, int lane) {
  const int32_t* p = col + lane;
  asm volatile("" : "+l"(p));
  return p;
}

template <bool kLinear, bool kHuge, int kB = kBatchLong>
__device__ __forceinline__ unsigned walk_long(const ChunkSmem& c, int t0, int t1,
                                              const PlanView& pv, int64_t ga) {
  static_assert(kB % 4 == 0, "batches of whole int4 reads");
  unsigned cnt = 0;
  const int lane = threadIdx.x & 31;
  const int32_t* colL = lane_base(pv.col, lane);
  int t = t0;
  for (; t + kB <= t1; t += kB) {
#if TC_L2PF
    // pull the key lines of the batch TC_L2PF batches ahead into L2 while this
    // batch's loads are outstanding: the loads in flight per lane are bounded
    // by registers, a prefetch holds none (lane u < kB takes tile u's first
    // line, lane kB + u its last)
    if (lane < 2 * kB && t + TC_L2PF * kB + (lane % kB) < t1) {
      const int q = lane % kB;
      const uint32_t x = (uint32_t)c.sT0[t + TC_L2PF * kB + q] + (lane >= kB ? 31u : 0u);
      asm volatile("prefetch.global.L2 [%0];" ::"l"(pv.col + x));
    }
#endif
    int32_t key[kB];
    load_batch<kB>(c, colL, t, key);
    int z[kB], zw[kB];
#pragma unroll
    for (int q = 0; q < kB; q += 4) {
      *reinterpret_cast<int4*>(z + q) = *reinterpret_cast<const int4*>(c.sT1 + t + q);
      *reinterpret_cast<int4*>(zw + q) = *reinterpret_cast<const int4*>(c.sT2 + t + q);
    }
    int zw_or = 0;  // first-lane fields are < 64, so the OR's code bits are the OR of the codes
#pragma unroll
    for (int u = 0; u < kB; ++u) zw_or |= zw[u];
    if ((zw_or >> 6) == 0) {
      // warp-uniform fast path, every tile of the batch probes a bitmap (most
      // batches: ~94% of RMAT keys meet a bitmap table): straight-line code,
      // no per-tile branch; zw is then just the first valid lane
#pragma unroll
      for (int u = 0; u < kB; ++u) {
        const unsigned word = (unsigned)c.sT0[(key[u] >> 5) + z[u]];
        const unsigned hit = (__funnelshift_r(word, 0u, (unsigned)key[u]) & 1u) ^ 1u;
        if (lane >= zw[u]) cnt += hit;
      }
    } else {
#pragma unroll
      for (int u = 0; u < kB; ++u) {
        const unsigned hit = probe_tile<kLinear, kHuge>(c, z[u], zw[u], key[u], lane, pv, ga);
        if (lane >= (zw[u] & 63)) cnt += hit;
      }
    }
  }
  for (; t < t1; t += 8) {  // tail: tiles past t1 repeat the last tile with every lane masked
    int z[8], zw[8];
    int32_t key[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) key[u] = __ldg(colL + (uint32_t)c.sT0[min(t + u, t1 - 1)]);
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int tt = min(t + u, t1 - 1);
      z[u] = c.sT1[tt];
      zw[u] = c.sT2[tt] | (t + u < t1 ? 0 : 32);  // first valid lane 32: none
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const unsigned hit = probe_tile<kLinear, kHuge>(c, z[u], zw[u], key[u], lane, pv, ga);
      if (lane >= (zw[u] & 63)) cnt += hit;
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
  int s = seg_of(c.sA, S, k0w);
  for (int k0 = k0w; k0 < k1w; k0 += 32 * kUnrollShort) {
    int seg[kUnrollShort];
#pragma unroll
    for (int u = 0; u < kUnrollShort; ++u) {
      const int t0 = k0 + 32 * u;
      const int j = s + 1 + lane;
      const int pos = (j <= S) ? c.sA[j] - t0 : 64;
      const unsigned bit = (pos >= 1 && pos <= 32) ? (1u << (pos - 1)) : 0u;
      const unsigned M = __reduce_or_sync(0xffffffffu, bit);
      seg[u] = s + __popc(M & below);
      s += __popc(M);
    }
    int32_t key[kUnrollShort];
    int gl[kUnrollShort];
#pragma unroll
    for (int u = 0; u < kUnrollShort; ++u) {
      const int k = k0 + 32 * u + lane;
      key[u] = -2;
      gl[u] = 0;
      if (k < k1w) {
        // col index sB + k < m < 2^32: a 32-bit add on the low word of sB
        // (two's complement wraps correctly) and one IMAD.WIDE
        const uint32_t lo = reinterpret_cast<const uint32_t*>(c.sB)[2 * seg[u]];
        key[u] = __ldg(pv.col + (lo + (uint32_t)k));
        gl[u] = c.sD[seg[u]];
      }
    }
#pragma unroll
    for (int u = 0; u < kUnrollShort; ++u) {
      // padding lanes have no table of their own: they must not probe (a
      // linear probe needs a table with an empty slot to terminate)
      if (k0 + 32 * u + lane >= k1w) continue;
      const int2 d = c.sInfo[gl[u]];
      if (kHuge && d.x < 0) {
        cnt += huge_probe(pv, ga + gl[u], key[u]);
      } else if (d.y <= 0) {
        // bitmap of the rank window: the trimmed key lies inside it (C-21),
        // so the word index (key >> 5) + code is in range
        const unsigned word = (unsigned)c.sHash[d.x + (key[u] >> 5) + d.y];
        cnt += (__funnelshift_r(word, 0u, (unsigned)key[u]) & 1u) ^ 1u;
      } else {
        cnt += table_probe<kLinear>(c.sHash + d.x, (uint32_t)d.y, key[u]);
      }
    }
  }
  return cnt;
}

template <bool kLinear, int kB = kBatchLong>
__device__ __forceinline__ unsigned consume(const ChunkSmem& c, const SlotHdr& h, int w0, int w1,
                                            const PlanView& pv) {
  if (h.is_long)
    return h.huge ? walk_long<kLinear, true, kB>(c, w0, w1, pv, h.ga)
                  : walk_long<kLinear, false, kB>(c, w0, w1, pv, h.ga);
  return h.huge ? walk_short<kLinear, true>(c, h.S, w0, w1, pv, h.ga)
                : walk_short<kLinear, false>(c, h.S, w0, w1, pv, h.ga);
}

// ------------------------------------------------------------------ support mode
// per-edge triangle counts.  A match of key w (at col
// position p_uw of u's suffix) in N+(v) closes the triangle {u, v, w}; its
// three edges are (u,v) (the segment's own CSR position), (u,w) = p_uw and
// (v,w) = row(v) + index of w in N+(v), which the support tables carry.

// Index of key in N+(v) through its support-mode table, or -1.
template <bool kLinear>
__device__ __forceinline__ int sup_find(const int* __restrict__ base, int off, int code,
                                        int32_t key) {
  if (code <= 0) {
    const int2 e = reinterpret_cast<const int2*>(base)[off + max((key >> 5) + code, 0)];
    const unsigned bits = ~(unsigned)e.x;
    const int b = key & 31;
    if (key < 0 || !((bits >> b) & 1u)) return -1;
    return e.y + __popc(bits & ((1u << b) - 1u));
  }
  const unsigned long long* H = reinterpret_cast<const unsigned long long*>(base) + off;
  const uint32_t n = (uint32_t)code;
  if (!kLinear) {
    const unsigned long long x1 = H[hash1(key, n)], x2 = H[hash2(key, n)];
    if ((int)(uint32_t)x1 == key) return (int)(x1 >> 32);
    if ((int)(uint32_t)x2 == key) return (int)(x2 >> 32);
    return -1;
  }
  uint32_t h = hash1(key, n);
  for (;;) {
    const unsigned long long x = H[h];
    if ((int)(uint32_t)x == key) return (int)(x >> 32);
    if ((int)(uint32_t)x < 0) return -1;
    h = (h + 1 == n) ? 0 : h + 1;
  }
}

// Index of key in the sorted list col[b, b+d), or -1 (huge tables).
__device__ __noinline__ int global_find(const int32_t* __restrict__ col, int64_t b, int64_t d,
                                        int32_t key) {
  int64_t lo = b, hi = b + d;
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (__ldg(col + mid) < key) lo = mid + 1; else hi = mid;
  }
  return (lo < b + d && __ldg(col + lo) == key) ? (int)(lo - b) : -1;
}

__device__ __forceinline__ int sup_lookup_any(const ChunkSmem& c, const PlanView& pv, int gl,
                                              int32_t key, bool linear) {
  const int2 info = c.sInfo[gl];
  if (info.x < 0)
    return global_find(pv.col, c.sGB[gl] + c.sGP[gl], c.sGP[gl + 1] - c.sGP[gl], key);
  return linear ? sup_find<true>(c.sHash, info.x, info.y, key)
                : sup_find<false>(c.sHash, info.x, info.y, key);
}

#ifndef TC_UNROLL_SUP
#define TC_UNROLL_SUP 5
#endif
constexpr int kUnrollSup = TC_UNROLL_SUP;  // tiles in flight per warp (support mode)
#ifndef TC_UNROLL_SUP_SHORT
#define TC_UNROLL_SUP_SHORT 3
#endif
constexpr int kUnrollSupShort = TC_UNROLL_SUP_SHORT;  // 32-key steps in flight (short class)
#ifndef TC_SUP_AGG
#define TC_SUP_AGG 1
#endif
#ifndef TC_SUP_FAST
#define TC_SUP_FAST 1
#endif

// Support-mode lookup of key in group gl's table; kHuge = the chunk has
// groups probed in global memory (otherwise that path is not compiled in).
template <bool kLinear, bool kHuge>
__device__ __forceinline__ int sup_lookup(const ChunkSmem& c, const PlanView& pv, int gl,
                                          uint32_t vrow, int32_t key) {
  const int2 info = c.sInfo[gl];
  if (kHuge && info.x < 0) return global_find(pv.col, vrow, c.sGP[gl + 1] - c.sGP[gl], key);
  return sup_find<kLinear>(c.sHash, info.x, info.y, key);
}

// col + lane / sup + lane in a register the compiler cannot see through.
__device__ __forceinline__ unsigned* lane_base_u(unsigned* p, int lane) {
  unsigned* q = p + lane;
  asm volatile("" : "+l"(q));
  return q;
}

// LONG class, support mode: tiles [t0, t1); a tile's lanes share one edge,
// whose count is warp-aggregated into one atomic.  Tile descriptors (see
// produce): sT0 = col position of the tile's first key, sT1 = row_ptr[v]
// (so (v, w) is sT1 + index of w in N+(v)), sT2 = the CSR position of the
// tile's own edge (u, v), sT3 = chunk-local group << 6 | valid lanes; every
// position < m < 2^32.
template <bool kLinear, bool kHuge>
__device__ __forceinline__ void walk_long_sup(const ChunkSmem& c, int t0, int t1,
                                              const PlanView& pv) {
  const int lane = threadIdx.x & 31;
  const int32_t* colL = lane_base(pv.col, lane);
  unsigned* supL = lane_base_u(pv.sup, lane);
#if TC_SUP_AGG
  // consecutive tiles of one long suffix share their edge (u, v): its count
  // is summed over the run and added once when the edge changes
  unsigned run = 0;
  uint32_t cur = 0u;
#endif
  for (int t = t0; t < t1; t += kUnrollSup) {
    int32_t key[kUnrollSup];
    uint32_t p[kUnrollSup], vr[kUnrollSup], own[kUnrollSup];
    int g6[kUnrollSup];
#pragma unroll
    for (int u = 0; u < kUnrollSup; ++u) {
      const int tt = min(t + u, t1 - 1);
      p[u] = (uint32_t)c.sT0[tt];
      vr[u] = (uint32_t)c.sT1[tt];
      own[u] = (uint32_t)c.sT2[tt];
      g6[u] = (t + u < t1) ? c.sT3[tt] : 0;
      key[u] = lane < (g6[u] & 63) ? __ldg(colL + p[u]) : -2;
    }
#if TC_SUP_FAST
    // warp-uniform fast path when every tile of the batch meets a bitmap
    // table (most batches on RMAT): all table reads issued before any use
    int2 inf[kUnrollSup];
    bool all_bm = true, no_huge = true;
#pragma unroll
    for (int u = 0; u < kUnrollSup; ++u) {
      inf[u] = c.sInfo[g6[u] >> 6];
      no_huge &= !kHuge || inf[u].x >= 0;
      all_bm &= inf[u].y <= 0;
    }
    all_bm &= no_huge;
    int idx[kUnrollSup];
    if (all_bm) {
      const int2* H2 = reinterpret_cast<const int2*>(c.sHash);
      int2 e[kUnrollSup];
#pragma unroll
      for (int u = 0; u < kUnrollSup; ++u) e[u] = H2[inf[u].x + max((key[u] >> 5) + inf[u].y, 0)];
#pragma unroll
      for (int u = 0; u < kUnrollSup; ++u) {
        const unsigned bits = ~(unsigned)e[u].x, b = (unsigned)key[u] & 31u;
        idx[u] = (key[u] >= 0 && ((bits >> b) & 1u)) ? e[u].y + __popc(bits & ((1u << b) - 1u)) : -1;
      }
    } else {
#pragma unroll
      for (int u = 0; u < kUnrollSup; ++u)
        idx[u] = key[u] >= 0 ? sup_lookup<kLinear, kHuge>(c, pv, g6[u] >> 6, vr[u], key[u]) : -1;
    }
#endif
#pragma unroll
    for (int u = 0; u < kUnrollSup; ++u) {
#if TC_SUP_FAST
      const int id = idx[u];
#else
      const int id = key[u] >= 0 ? sup_lookup<kLinear, kHuge>(c, pv, g6[u] >> 6, vr[u], key[u]) : -1;
#endif
      const unsigned bal = __ballot_sync(0xffffffffu, id >= 0);
      if (id >= 0) {
        atomicAdd(supL + p[u], 1u);                       // (u, w)
        atomicAdd(pv.sup + (vr[u] + (uint32_t)id), 1u);   // (v, w)
      }
#if TC_SUP_AGG
      if (own[u] != cur) {
        if (lane == 0 && run) atomicAdd(pv.sup + cur, run);  // (u, v)
        run = 0;
        cur = own[u];
      }
      run += (unsigned)__popc(bal);
#else
      if (lane == 0 && bal) atomicAdd(pv.sup + own[u], (unsigned)__popc(bal));  // (u, v)
#endif
    }
  }
#if TC_SUP_AGG
  if (lane == 0 && run) atomicAdd(pv.sup + cur, run);  // (u, v)
#endif
}

// SHORT class, support mode: flat keys [k0w, k1w) of the chunk.
__device__ __forceinline__ void walk_short_sup(const ChunkSmem& c, int S, int k0w, int k1w,
                                               const PlanView& pv, bool linear) {
  auto load = [&](int sg, int k) { return __ldg(pv.col + c.sB[sg] + k); };
  warp_walk<kUnrollSupShort>(c.sA, S, k0w, k1w, load, [&](int sg, int k, int32_t key) {
    const int gl = c.sD[sg];
    const int idx = sup_lookup_any(c, pv, gl, key, linear);
    if (idx >= 0) {
      atomicAdd(pv.sup + c.sB[sg] + k, 1u);                  // (u, w)
      atomicAdd(pv.sup + c.sGB[gl] + c.sGP[gl] + idx, 1u);   // (v, w)
      atomicAdd(pv.sup + c.sE[sg], 1u);                      // (u, v)
    }
  });
}

// ------------------------------------------------------------------ producers
// Stage chunk cix into a slot and build its tables.  pt = producer thread id
// in [0, PT); the PT producer threads synchronise on named barrier 1.  The
// header is written by producer 0 before its own mbarrier arrive, so the
// consumers see it once every producer has arrived.
template <int kB, bool kSup = false>
__device__ __forceinline__ void produce(const PlanView& pv, int64_t cix, int64_t e_begin,
                                        int64_t e_end, unsigned char* region, SlotHdr& hdr,
                                        int pt, int PT, int bar = 1) {
  const int64_t sa = max(__ldg(pv.chunk_seg + (cix)), e_begin), sb = min(__ldg(pv.chunk_seg + (cix + 1)), e_end);
  if (sa >= sb) {  // empty after clipping to the range
    if (pt == 0) {
      hdr.S = 0;
      hdr.done = 0;
    }
    return;
  }
  const bool is_long = cix < pv.n_long_chunks;
  const int S = (int)(sb - sa);
  const int64_t ga = __ldg(pv.seg_group + (sa)), gb = (int64_t)__ldg(pv.seg_group + (sb - 1)) + 1;
  const int G = (int)(gb - ga);
  const int64_t slot0 = __ldg(pv.slot_prefix + (ga));
  const int nslots = (int)(__ldg(pv.slot_prefix + (gb)) - slot0);
  // key_prefix is mod 2^32: chunk-relative differences are exact (< 2^32)
  const uint32_t kp0 = __ldg(pv.key_prefix + (sa));
  const int T = is_long ? (int)((__ldg(pv.key_prefix + (sb)) - kp0) >> 5) : 0;
  ChunkSmem c = kSup ? slot_view_sup(region, S, G, T, nslots) : slot_view(region, S, G, T);

  // 1. stage edges and groups; empty slots.  Each producer thread handles
  //    kB items per batch with all their global loads issued before any
  //    store, so a batch costs one memory latency.
  for (int base = pt; base <= S; base += PT * kB) {
    uint32_t kp[kB], st[kB];
    int ln[kB], gr[kB];
#pragma unroll
    for (int r = 0; r < kB; ++r) {
      const int i = base + r * PT;
      kp[r] = 0;
      st[r] = 0;
      ln[r] = gr[r] = 0;
      if (i <= S) kp[r] = __ldg(pv.key_prefix + (sa + i));
      if (i < S) {
        st[r] = __ldg(pv.seg_start + (sa + i));
        ln[r] = __ldg(pv.seg_len + (sa + i));
        gr[r] = __ldg(pv.seg_group + (sa + i));
      }
    }
#pragma unroll
    for (int r = 0; r < kB; ++r) {
      const int i = base + r * PT;
      const int rel = (int)(kp[r] - kp0);  // u32 arithmetic
      if (i <= S) c.sA[i] = is_long ? (rel >> 5) : rel;
      if (i < S) {
        c.sB[i] = is_long ? (int64_t)st[r] : (int64_t)st[r] - rel;
        c.sC[i] = ln[r];
        c.sD[i] = gr[r] - (int)ga;
#if TC_PF_SHORT
        // short class: pull the edge's keys (< 32, at most two lines) into L2
        // now; the walk reads them after the tables are built
        if (!is_long && !kSup) {
          const int32_t* k0 = pv.col + st[r];
          asm volatile("prefetch.global.L2 [%0];" ::"l"(k0));
          if (((uintptr_t)k0 & 127) + 4 * (uintptr_t)ln[r] > 128)
            asm volatile("prefetch.global.L2 [%0];" ::"l"(k0 + ln[r] - 1));
        }
#endif
      }
    }
  }
  if (kSup)
    for (int i = pt; i < S; i += PT) c.sE[i] = __ldg(pv.seg_edge + (sa + i));
  const int64_t ip0 = __ldg(pv.ins_prefix + (ga));
  int huge = 0;
  for (int base = pt; base <= G; base += PT * kB) {
    int64_t ip[kB], sp[kB], sp1[kB], ib[kB];
    int cd[kB];
#pragma unroll
    for (int r = 0; r < kB; ++r) {
      const int i = base + r * PT;
      ip[r] = sp[r] = sp1[r] = ib[r] = 0;
      cd[r] = 0;
      if (i <= G) ip[r] = __ldg(pv.ins_prefix + (ga + i));
      if (i < G) {
        sp[r] = __ldg(pv.slot_prefix + (ga + i));
        sp1[r] = __ldg(pv.slot_prefix + (ga + i + 1));
        ib[r] = __ldg(pv.grp_ibase + (ga + i));
        cd[r] = __ldg(pv.grp_code + (ga + i));
      }
    }
#pragma unroll
    for (int r = 0; r < kB; ++r) {
      const int i = base + r * PT;
      if (i <= G) c.sGP[i] = (int)(ip[r] - ip0);
      if (i < G) {
        const int ns = (int)(sp1[r] - sp[r]);
        c.sInfo[i] = ns > 0 ? make_int2((int)(sp[r] - slot0), cd[r]) : make_int2(-1, 0);
        huge |= ns == 0;
        c.sGB[i] = ib[r] + ip0;  // row start - chunk-relative insert prefix
      }
    }
  }
  {
    // support mode: 8-B entries -> twice the words (nslots is a multiple of 4)
    const int nwords = kSup ? 2 * nslots : nslots;
    int4* h4 = reinterpret_cast<int4*>(c.sHash);
    for (int i = pt; i < (nwords >> 2); i += PT) h4[i] = make_int4(-1, -1, -1, -1);
    for (int i = (nwords & ~3) + pt; i < nwords; i += PT) c.sHash[i] = -1;
  }
  const int any_huge = named_sync_or(bar, PT, huge);

  // 2. long class: one descriptor per 32-key tile (producer thread per edge)
  if (is_long) {
    for (int i = pt; i < S; i += PT) {
      const int ts = c.sA[i], te = c.sA[i + 1], len = c.sC[i], gl = c.sD[i];
      const int2 d = c.sInfo[gl];
      const int toff = d.x >= 0 ? d.x : -1 - gl;
      const int64_t st = c.sB[i];
      for (int t = ts; t < te; ++t) {
        const int64_t p = st + ((int64_t)(t - ts) << 5);
        const int lanes = min(32, len - ((t - ts) << 5));
        // support mode: the tile names its edge (chunk-local) instead of its table
        if (kSup) {  // walk_long_sup's descriptor (positions < m < 2^32)
          c.sT0[t] = (int)(uint32_t)p;
          c.sT1[t] = (int)(uint32_t)(c.sGB[gl] + c.sGP[gl]);  // row_ptr[v]
          c.sT2[t] = (int)(uint32_t)c.sE[i];
          c.sT3[t] = (gl << 6) | lanes;
        } else {
          // walk_long: a partial last tile is shifted back to the edge's last 32
          // keys (len >= 32 in the long class), its first 32 - lanes lanes
          // masked.  sT1 = z, sT2 = (code << 5) | first valid lane, code:
          // bitmap 0 (z = word base), hash = slots (z = offset), huge -1.
          // (6-bit lane field: 32 = no valid lane)
          c.sT0[t] = (int)(uint32_t)(p - (32 - lanes));
          const int zt = d.x < 0 ? toff : (int)(c.sHash - c.sT0) + (d.y <= 0 ? d.x + d.y : d.x);
          const int zwt = ((d.x < 0 ? -1 : (d.y <= 0 ? 0 : d.y)) * 64) | (32 - lanes);
          c.sT1[t] = zt;
          c.sT2[t] = zwt;
        }
      }
    }
  }

  // 3. hash N+(v) of every group touched by the chunk (flattened over groups,
  //    kInsU tiles of N+(v) loads in flight per producer lane)
#ifndef TC_INS_UNROLL
#define TC_INS_UNROLL 4
#endif
  constexpr int kInsU = kB >= 4 ? TC_INS_UNROLL : 4;  // N+(v) row loads in flight per producer lane (long-class producers; the flat kernel keeps 4)
  const int pw = pt >> 5, npw = PT >> 5;
  const int NI = c.sGP[G];
  const int i0 = (int)((unsigned)NI * (unsigned)pw / (unsigned)npw),
            i1 = (int)((unsigned)NI * (unsigned)(pw + 1) / (unsigned)npw);  // NI * npw < 2^31
  auto load_row = [&](int g, int k) { return __ldg(pv.col + c.sGB[g] + k); };
  // short class: linear probing from the start when the plan says so (its
  // tables are tiny — a few keys each — and a chunk whose cuckoo insert fails
  // builds all its tables twice)
  bool linear = pv.probe_mode == 1 || (!is_long && pv.short_linear);
  if constexpr (kSup) {
    // Support mode: entries carry the key's index j in N+(v) (its edge (v,w)
    // is col position row(v) + j).  Bitmap word x = {bits, members of N+(v)
    // in words before x}: the inserter of the first key of each word writes
    // the count of the words it opens (those after its predecessor's word).
    auto ins_sup = [&](int g, int k, int32_t key, bool lin) {
      const int2 d = c.sInfo[g];
      if (d.x < 0) return;
      const int j = k - c.sGP[g];
      if (d.y <= 0) {
        int2* W = reinterpret_cast<int2*>(c.sHash) + d.x;
        const int w = (key >> 5) + d.y;
        atomicAnd(&W[w].x, ~(1 << (key & 31)));
        const int pw = j > 0 ? (__ldg(pv.col + c.sGB[g] + k - 1) >> 5) + d.y : -1;
        for (int x = pw + 1; x <= w; ++x) W[x].y = j;
      } else {
        unsigned long long* H = reinterpret_cast<unsigned long long*>(c.sHash) + d.x;
        const unsigned long long e = ((unsigned long long)(uint32_t)j << 32) | (uint32_t)key;
        if (lin) linear_insert64(H, (uint32_t)d.y, key, e);
        else if (!cuckoo_insert64(H, (uint32_t)d.y, key, e, pv.max_kicks)) linear = true;  // flag, below
      }
    };
    const bool want_linear = linear;
    linear = false;
    warp_walk<kInsU>(c.sGP, G, i0, i1, load_row,
                     [&](int g, int k, int32_t key) { ins_sup(g, k, key, want_linear); });
    if (!want_linear && named_sync_or(bar, PT, linear)) {  // a cuckoo insert failed
      if (pt == 0) atomicAdd(&g_counters[0], 1ull);
      for (int i = pt; i < 2 * nslots; i += PT) c.sHash[i] = -1;
      named_sync(bar, PT);
      warp_walk<kInsU>(c.sGP, G, i0, i1, load_row,
                       [&](int g, int k, int32_t key) { ins_sup(g, k, key, true); });
      linear = true;
    }
    linear = linear || want_linear;
  } else {
  auto insert_linear = [&](int g, int, int32_t key) {
    const int2 d = c.sInfo[g];
    if (d.x < 0) return;
    if (d.y <= 0) bitmap_insert(c.sHash + d.x, d.y, key);
    else linear_insert(c.sHash + d.x, (uint32_t)d.y, key);
  };
  if (linear) {
    warp_walk<kInsU>(c.sGP, G, i0, i1, load_row, insert_linear);
  } else {
    bool ok = true;
    warp_walk<kInsU>(c.sGP, G, i0, i1, load_row, [&](int g, int, int32_t key) {
      const int2 d = c.sInfo[g];
      if (d.x < 0) return;
      if (d.y <= 0) bitmap_insert(c.sHash + d.x, d.y, key);
      else if (!cuckoo_insert(c.sHash + d.x, (uint32_t)d.y, key, pv.max_kicks)) ok = false;
    });
    if (named_sync_or(bar, PT, !ok)) {  // uniform over producers: rebuild with linear probing
      if (pt == 0) atomicAdd(&g_counters[0], 1ull);
      linear = true;
      for (int i = pt; i < nslots; i += PT) c.sHash[i] = -1;
      named_sync(bar, PT);
      warp_walk<kInsU>(c.sGP, G, i0, i1, load_row, insert_linear);
    }
  }
  }
  if (pt == 0) {
    hdr.sa = sa;
    hdr.ga = ga;
    hdr.S = S;
    hdr.G = G;
    hdr.T = T;
    hdr.nslots = nslots;
    hdr.is_long = is_long;
    hdr.linear = linear;
    hdr.done = 0;
    hdr.huge = any_huge;
    hdr.next = 0;
  }
}

// kBlock: the launch bound (1024 threads cap a thread at 64 registers, which
// bounds the key loads in flight to kB = 8 tiles per lane; smaller CTAs buy
// registers for deeper batches: Tuning::batch, block_threads).
template <int kBlock, int kB>
__global__ void __launch_bounds__(kBlock, 1)
    k_count(PlanView pv, int64_t c_begin, int64_t c_end, int64_t e_begin, int64_t e_end,
            int64_t slot_bytes, Tuning tu, unsigned long long* __restrict__ out,
            const FuseArgs fuse) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ unsigned long long red[kMaxBlock / 32];
  __shared__ __align__(8) uint64_t full_bar[kMaxSlots];
  __shared__ __align__(8) uint64_t empty_bar[kMaxSlots];
  __shared__ SlotHdr hdr[kMaxSlots];
  const int warp = threadIdx.x >> 5, nw = blockDim.x >> 5, lane = threadIdx.x & 31;
  const int n_prod = max(1, min(nw - 1, nw / tu.prod_div)), n_cons = nw - n_prod;
  const int PT = n_prod * 32;
  const int nslots = tu.slots;
  const uint32_t hint = (uint32_t)tu.wait_hint_ns;
  // producer groups (Tuning::prod_groups): group g fills the CTA's chunks
  // k = g, g + ng, ... into slot k mod nslots, on its own named barrier, so
  // ng chunks are in production at once (a chunk's staging and table build
  // are latency-bound where its tables are many and small)
  const int ng = max(1, min(tu.prod_groups, n_prod));
  const int gsz = n_prod / ng, PTg = gsz * 32;
  if (threadIdx.x == 0) {
    for (int i = 0; i < nslots; ++i) {
      mbar_init(&full_bar[i], PTg);      // every thread of the filling group arrives
      mbar_init(&empty_bar[i], n_cons);  // one lane per consumer warp
    }
  }
  __syncthreads();

  unsigned long long acc = 0;
  if (warp < n_prod) {
    // ------------------------------------------------------------ producers
    const int g = warp / gsz;
    if (warp < ng * gsz) {  // (warps beyond ng * gsz, if n_prod is odd, idle)
      const int pt = threadIdx.x - g * PTg;
      // slot / fill number kept incrementally (no 64-bit division per chunk)
      int slot = g;
      uint32_t j = 0;  // fill number of this slot
      // This CTA's chunks are c_begin + b + k * grid; this group's k = g + i * ng.
      // (Taking them alternately from both ends of the range, to mix the
      // table-heavy head with the probe-heavy tail, measured slower: C3 44.4
      // -> 45.4 ms, C4 558 -> 575, profiles/r5a_*.)
      for (int64_t k = g;; k += ng) {
        const int64_t cix = c_begin + blockIdx.x + k * gridDim.x;
        if (j > 0) wait_empty(&empty_bar[slot], (j - 1) & 1, hint);
        if (cix >= c_end) {
          if (pt == 0) hdr[slot].done = 1;
          mbar_arrive(&full_bar[slot]);
          break;
        }
        produce<4>(pv, cix, e_begin, e_end, smem + slot * slot_bytes, hdr[slot], pt, PTg, 1 + g);
        mbar_arrive(&full_bar[slot]);
        slot += ng;
        if (slot >= nslots) {
          slot -= nslots;
          ++j;
        }
      }
    }
  } else {
    // ------------------------------------------------------------ consumers
    const int cw = warp - n_prod;
    int slot = 0;
    uint32_t fill = 0;
    for (;; slot = (slot + 1 == nslots) ? (++fill, 0) : slot + 1) {
      wait_full(&full_bar[slot], fill & 1u, hint);
      const SlotHdr h = hdr[slot];
      if (h.done) break;
      if (h.S > 0) {
        const ChunkSmem c = slot_view(smem + slot * slot_bytes, h.S, h.G, h.T);
        const int NU = h.is_long ? h.T : c.sA[h.S];
        const int grab = h.is_long ? tu.grab_long : tu.grab_short;
        if (grab <= 0) {  // static split: a contiguous share per consumer warp
          // 32-bit: NU * n_cons < 2^31 (a chunk slot holds < 2^16 tiles / keys)
          int w0 = (int)((unsigned)NU * (unsigned)cw / (unsigned)n_cons),
              w1 = (int)((unsigned)NU * (unsigned)(cw + 1) / (unsigned)n_cons);
          if (h.is_long) {  // walk_long batches start at multiples of 8 tiles
            w0 = min((w0 + 7) & ~7, NU);
            w1 = cw + 1 == n_cons ? NU : min((w1 + 7) & ~7, NU);
          }
          acc += h.linear ? consume<true, kB>(c, h, w0, w1, pv) : consume<false, kB>(c, h, w0, w1, pv);
        } else {  // dynamic: grab `grab` units at a time from the slot's counter
          for (;;) {
            int w0 = 0;
            if (lane == 0) w0 = atomicAdd(&hdr[slot].next, grab);
            w0 = __shfl_sync(0xffffffffu, w0, 0);
            if (w0 >= NU) break;
            const int w1 = min(w0 + grab, NU);
            acc += h.linear ? consume<true, kB>(c, h, w0, w1, pv) : consume<false, kB>(c, h, w0, w1, pv);
          }
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty_bar[slot]);
    }
  }

  // u64 reduction: warp shuffle -> CTA -> one atomic
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_down_sync(0xffffffffu, acc, o);
  if (lane == 0) red[warp] = acc;
  __syncthreads();
  if (warp == 0) {
    unsigned long long v = lane < nw ? red[lane] : 0ull;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
    if (lane == 0) {
      if (v) atomicAdd(out, v);
      if (fuse.own) fused_epilogue(out, fuse);  // f4: the last CTA sums across ranks
    }
  }
}

// The long-class kernel's instances: (launch bound, tiles per batch).
const void* const kCountKernels[] = {
    (const void*)k_count<1024, 8>, (const void*)k_count<768, 8>, (const void*)k_count<768, 12>,
    (const void*)k_count<768, 16>, (const void*)k_count<512, 16>, (const void*)k_count<512, 24>};

// The instance for a block size and batch (Tuning::batch; 0 = the default 8):
// block > 768 or an unknown pair runs the 1024-bound, 8-tile instance.
const void* count_kernel(int block, int batch) {
  if (block <= 512) return batch >= 24 ? kCountKernels[5] : kCountKernels[4];
  if (block <= 768) return batch >= 16 ? kCountKernels[3] : batch >= 12 ? kCountKernels[2] : kCountKernels[1];
  return kCountKernels[0];
}

// SHORT-class chunks: every warp stages, builds and probes (no producer /
// consumer split: a short chunk's table building is as much work as its
// probing), one chunk slot per CTA and 3 CTAs per SM so that one CTA's
// staging and building latency overlaps the others' probing.
__global__ void __launch_bounds__(kFlatBlock, kFlatCTAs)
    k_count_flat(PlanView pv, int64_t c_begin, int64_t c_end, int64_t e_begin, int64_t e_end,
                 unsigned long long* __restrict__ out, const FuseArgs fuse) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ unsigned long long red[kFlatBlock / 32];
  __shared__ SlotHdr hdr;
  const int warp = threadIdx.x >> 5, nw = blockDim.x >> 5, lane = threadIdx.x & 31;
  unsigned long long acc = 0;
  for (int64_t cix = c_begin + blockIdx.x; cix < c_end; cix += gridDim.x) {
    produce<2>(pv, cix, e_begin, e_end, smem, hdr, threadIdx.x, blockDim.x);
    __syncthreads();
    const SlotHdr h = hdr;
    if (h.S > 0) {
      const ChunkSmem c = slot_view(smem, h.S, h.G, h.T);  // short class only: T = 0
      const int NU = c.sA[h.S];
      const int w0 = (int)((unsigned)NU * (unsigned)warp / (unsigned)nw),
                w1 = (int)((unsigned)NU * (unsigned)(warp + 1) / (unsigned)nw);
      if (h.linear)
        acc += h.huge ? walk_short<true, true>(c, h.S, w0, w1, pv, h.ga)
                      : walk_short<true, false>(c, h.S, w0, w1, pv, h.ga);
      else
        acc += h.huge ? walk_short<false, true>(c, h.S, w0, w1, pv, h.ga)
                      : walk_short<false, false>(c, h.S, w0, w1, pv, h.ga);
    }
    __syncthreads();  // the slot is rebuilt by the next chunk
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_down_sync(0xffffffffu, acc, o);
  if (lane == 0) red[warp] = acc;
  __syncthreads();
  if (warp == 0) {
    unsigned long long v = lane < nw ? red[lane] : 0ull;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
    if (lane == 0) {
      if (v) atomicAdd(out, v);
      if (fuse.own) fused_epilogue(out, fuse);  // f4: the last CTA sums across ranks
    }
  }
}

// Support mode kernel: one chunk at a time per CTA, all warps build then
// all warps probe (both classes; 8-B table entries double the SMEM of a chunk).
__global__ void __launch_bounds__(kMaxBlock, 1)
    k_support(PlanView pv, int64_t c_begin, int64_t c_end) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ SlotHdr hdr;
  const int warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  for (int64_t cix = c_begin + blockIdx.x; cix < c_end; cix += gridDim.x) {
    produce<2, true>(pv, cix, 0, INT64_MAX, smem, hdr, threadIdx.x, blockDim.x);
    __syncthreads();
    const SlotHdr h = hdr;
    if (h.S > 0) {
      const ChunkSmem c = slot_view_sup(smem, h.S, h.G, h.T, h.nslots);
      const int NU = h.is_long ? h.T : c.sA[h.S];
      const int w0 = (int)((unsigned)NU * (unsigned)warp / (unsigned)nw),
                w1 = (int)((unsigned)NU * (unsigned)(warp + 1) / (unsigned)nw);
      if (h.is_long) {
        if (h.huge)
          h.linear ? walk_long_sup<true, true>(c, w0, w1, pv) : walk_long_sup<false, true>(c, w0, w1, pv);
        else
          h.linear ? walk_long_sup<true, false>(c, w0, w1, pv) : walk_long_sup<false, false>(c, w0, w1, pv);
      }
      else if (w0 < w1) walk_short_sup(c, h.S, w0, w1, pv, h.linear);
    }
    __syncthreads();  // the slot is rebuilt by the next chunk
  }
}

// Largest i in [0, len) with a[i] <= x (a non-decreasing, a[0] <= x).
__device__ __forceinline__ int64_t last_le(const int64_t* __restrict__ a, int64_t len, int64_t x) {
  int64_t lo = 0, hi = len - 1;
  while (lo < hi) {
    const int64_t mid = (lo + hi + 1) >> 1;
    if (a[mid] <= x) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// CSR position of every live segment's own edge (u,v): u = the row holding
// its suffix, v = the head whose row starts at grp_ibase + ins_prefix, and
// (u,v) = the position of v in N+(u), which precedes the suffix.
__global__ void k_seg_edge(const int64_t* __restrict__ row_ptr, int64_t n,
                           const int32_t* __restrict__ col, const uint32_t* __restrict__ seg_start,
                           const int32_t* __restrict__ seg_group,
                           const int64_t* __restrict__ grp_ibase,
                           const int64_t* __restrict__ ins_prefix, int64_t S,
                           int64_t* __restrict__ seg_edge) {
  for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < S;
       s += (int64_t)gridDim.x * blockDim.x) {
    const int64_t st = (int64_t)seg_start[s];
    const int g = seg_group[s];
    const int64_t u = last_le(row_ptr, n + 1, st);
    const int32_t v = (int32_t)last_le(row_ptr, n + 1, grp_ibase[g] + ins_prefix[g]);
    int64_t lo = row_ptr[u], hi = st;
    while (lo < hi) {
      const int64_t mid = (lo + hi) >> 1;
      if (col[mid] < v) lo = mid + 1; else hi = mid;
    }
    seg_edge[s] = lo;
  }
}

// Original ids of every CSR edge: (perm[row(p)], perm[col[p]]).
__global__ void k_edge_ends(const int64_t* __restrict__ row_ptr, int64_t n,
                            const int32_t* __restrict__ col, const int32_t* __restrict__ perm,
                            int64_t m, int32_t* __restrict__ eu, int32_t* __restrict__ ev) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < m;
       p += (int64_t)gridDim.x * blockDim.x) {
    eu[p] = perm[last_le(row_ptr, n + 1, p)];
    ev[p] = perm[col[p]];
  }
}


int optin_smem() {
  int dev = 0, v = 0;
  TC_CUDA(cudaGetDevice(&dev));
  TC_CUDA(cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  return v;
}

int static_smem(const void* f) {
  cudaFuncAttributes fa;
  TC_CUDA(cudaFuncGetAttributes(&fa, f));
  return (int)fa.sharedSizeBytes;
}

// cudaFuncSetAttribute applies to the current device's context: the flag is
// per device (graphs may be built on several devices of one process), and
// set at most once per device even with concurrent callers.
constexpr int kMaxDevices = 64;
std::once_flag g_attr_once[kMaxDevices];

void set_attr() {
  for (const void* f : kCountKernels)
    TC_CUDA(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 optin_smem() - static_smem(f)));
  TC_CUDA(cudaFuncSetAttribute(k_count_flat, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               optin_smem() - static_smem((const void*)k_count_flat)));
  TC_CUDA(cudaFuncSetAttribute(k_support, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               optin_smem() - static_smem((const void*)k_support)));
}

void ensure_attr() {
  int dev = 0;
  TC_CUDA(cudaGetDevice(&dev));
  if (dev < 0 || dev >= kMaxDevices) {  // beyond the table: set it every time (cheap)
    set_attr();
    return;
  }
  std::call_once(g_attr_once[dev], set_attr);  // a throw leaves the flag unset
}

int64_t slot_bytes_of(int64_t need) { return (need + 15) & ~int64_t(15); }

PlanView plan_view(const tc_graph* g) {
  const Plan& P = g->plan;
  PlanView pv;
  pv.col = g->col.get();
  pv.key_prefix = P.key_prefix.get();
  pv.seg_start = P.seg_start.get();
  pv.seg_len = P.seg_len.get();
  pv.seg_group = P.seg_group.get();
  pv.ins_prefix = P.ins_prefix.get();
  pv.grp_ibase = P.grp_ibase.get();
  pv.slot_prefix = P.slot_prefix.get();
  pv.grp_code = P.grp_code.get();
  pv.chunk_seg = P.chunk_seg.get();
  pv.n_long_chunks = P.n_long_chunks;
  pv.probe_mode = P.opt.probe_mode;
  pv.short_linear = P.tune.short_linear;
  pv.seg_edge = nullptr;
  pv.sup = nullptr;
  pv.max_kicks = P.tune.max_kicks;
  pv.m = g->m;
  return pv;
}

}  // namespace

void read_counters(uint64_t* h, bool reset) {
  TC_CUDA(cudaMemcpyFromSymbol(h, g_counters, sizeof(unsigned long long) * 4));
  if (reset) {
    const unsigned long long z[4] = {0, 0, 0, 0};
    TC_CUDA(cudaMemcpyToSymbol(g_counters, z, sizeof(z)));
  }
}

int num_sms() {
  int dev = 0, v = 0;
  TC_CUDA(cudaGetDevice(&dev));
  TC_CUDA(cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev));
  return v;
}

int max_smem_per_block() { return optin_smem() - static_smem(kCountKernels[0]); }

int max_chunk_smem(const Tuning& tu) { return (max_smem_per_block() / tu.slots) & ~15; }

// One chunk of the flat kernel must leave room for 3 CTAs per SM.
int max_flat_chunk_smem() {
  int dev = 0, per_sm = 0;
  TC_CUDA(cudaGetDevice(&dev));
  TC_CUDA(cudaDeviceGetAttribute(&per_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev));
  const int per_cta = per_sm / kFlatCTAs - 1024 - static_smem((const void*)k_count_flat);  // 1 KB reserved per CTA
  return std::min(per_cta, optin_smem() - static_smem((const void*)k_count_flat)) & ~15;
}

int count_occupancy(int block, int64_t smem_bytes, const Tuning& tu) {
  ensure_attr();
  int occ = 0;
  TC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(
      &occ, count_kernel(block, tu.batch), block, (size_t)(tu.slots * slot_bytes_of(smem_bytes))));
  return occ;
}

int flat_occupancy(int64_t smem_bytes) {
  ensure_attr();
  int occ = 0;
  TC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_count_flat, kFlatBlock,
                                                        (size_t)slot_bytes_of(smem_bytes)));
  return occ;
}

int count_chunks(const tc_graph* g, int64_t c_begin, int64_t c_end, int64_t e_begin,
                 int64_t e_end, cudaStream_t s, unsigned long long* d_out, const FuseArgs* fuse) {
  TC_CUDA(cudaMemsetAsync(d_out, 0, sizeof(unsigned long long), s));
  const Plan& P = g->plan;
  if (c_end <= c_begin || e_end <= e_begin) return 0;
  ensure_attr();
  const PlanView pv = plan_view(g);
  FuseArgs none;
  memset(&none, 0, sizeof(none));
  // long-class chunks [c_begin, min(c_end, nL)): warp-specialised kernel;
  // short-class chunks: flat kernel.  The last launch carries the fused sum.
  const int64_t l0 = c_begin, l1 = std::min(c_end, P.n_long_chunks);
  const int64_t s0 = std::max(c_begin, P.n_long_chunks), s1 = c_end;
  int launched = 0;
  if (l1 > l0) {
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(l1 - l0, P.grid));
    const int64_t sb = slot_bytes_of(P.smem_bytes);
    const FuseArgs& fa = (fuse && s1 <= s0) ? *fuse : none;  // no later launch follows
    void* args[] = {(void*)&pv, (void*)&l0, (void*)&l1, (void*)&e_begin, (void*)&e_end,
                    (void*)&sb, (void*)&P.tune, (void*)&d_out, (void*)&fa};
    TC_CUDA(cudaLaunchKernel(count_kernel(P.block, P.tune.batch), dim3(grid), dim3(P.block), args,
                             (size_t)(P.tune.slots * sb), s));
    ++launched;
  }
  if (s1 > s0) {
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(s1 - s0, P.grid_flat));
    k_count_flat<<<grid, kFlatBlock, (size_t)slot_bytes_of(P.smem_flat), s>>>(
        pv, s0, s1, e_begin, e_end, d_out, fuse ? *fuse : none);
    TC_LAUNCH();
    ++launched;
  }
  return launched;
}

void support_all(const tc_graph* g, cudaStream_t s, unsigned* d_sup) {
  if (g->m > 0) TC_CUDA(cudaMemsetAsync(d_sup, 0, sizeof(unsigned) * (size_t)g->m, s));
  const Plan& P = g->plan;
  if (P.S == 0 || P.n_chunks == 0) return;
  ensure_attr();
  DevBuf<int64_t> seg_edge(P.S, s);
  const int grid_e = (int)std::min<int64_t>((P.S + 255) / 256, 148 * 16);
  k_seg_edge<<<grid_e, 256, 0, s>>>(g->row_ptr.get(), g->n, g->col.get(), P.seg_start.get(),
                                    P.seg_group.get(), P.grp_ibase.get(), P.ins_prefix.get(), P.S,
                                    seg_edge.get());
  TC_LAUNCH();
  PlanView pv = plan_view(g);
  pv.seg_edge = seg_edge.get();
  pv.sup = d_sup;
  // a chunk's support layout is at most twice its count layout (tc_count.cu
  // slot_view_sup: + 4 B per table word + 8 B per edge)
  const int64_t bytes = slot_bytes_of(2 * std::max(P.smem_bytes, P.smem_flat) + 16);
  if (bytes > optin_smem() - static_smem((const void*)k_support))
    fail(TC_ERR_UNSUPPORTED, "support tables exceed shared memory (lower huge_degree)");
  int occ = 0;
  TC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_support, kMaxBlock, (size_t)bytes));
  if (occ < 1) fail(TC_ERR_UNSUPPORTED, "support kernel cannot launch");
  const int grid = (int)std::min<int64_t>(P.n_chunks, (int64_t)occ * num_sms());
  k_support<<<grid, kMaxBlock, (size_t)bytes, s>>>(pv, 0, P.n_chunks);
  TC_LAUNCH();
}

void edge_ends(const tc_graph* g, cudaStream_t s, int32_t* d_u, int32_t* d_v) {
  if (g->m == 0) return;
  const int grid = (int)std::min<int64_t>((g->m + 255) / 256, 148 * 16);
  k_edge_ends<<<grid, 256, 0, s>>>(g->row_ptr.get(), g->n, g->col.get(), g->perm.get(), g->m, d_u,
                                   d_v);
  TC_LAUNCH();
}

}  // namespace tc

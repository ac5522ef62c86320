// tc_fused.cuh — SURVEY.md §8(f) row f4: the cross-GPU sum of the partial
// counts over NVLink peer memory, as a device function shared by the count
// kernels' last-CTA epilogue (tc_count.cu) and the stand-alone finishing
// kernel of an empty range (tc_fused.cu).
//
// Symmetric buffer (same layout on every rank, zero-initialised once):
//   word[0], word[1]  sum of the epochs with parity 0 / 1   (every replica)
//   word[2]           arrivals, world per epoch               (every replica)
//   word[3]           POISON: set by this rank when a peer never arrived
//   word[4]           grid-completion ticket of the count kernel (local)
// Protocol for epoch e (slot = e & 1), run by ONE thread after the rank's
// partial is final:
//   1. clear this rank's replica of the OTHER slot, fence;
//   2. add the partial into slot on every replica — one multimem.red through
//      the NVLS multicast address, or one red per peer over NVLink P2P;
//   3. fence, then add 1 to the arrivals of every replica (release);
//   4. spin (acquire) until the own arrivals reach world * e;
//   5. T = own slot.
// Epoch-parity double buffering is safe: rank r clears slot (e+1)&1 before it
// arrives in epoch e, and no rank adds into that slot (in epoch e+1) before
// it has seen every arrival of epoch e.  A peer that never arrives within
// kArrivalTimeoutNs sets the POISON word and yields UINT64_MAX instead of
// hanging the stream; the buffer must then be recreated (the late partial may
// still land in it).
#pragma once
#include "tc.h"

namespace tc {

constexpr unsigned long long kArrivalTimeoutNs = 20ull * 1000 * 1000 * 1000;  // 20 s
constexpr int kFusedWords = 8;  // u64 words of the symmetric buffer (>= 5 used)

struct FuseArgs {
  unsigned long long* own;  // this rank's unicast address of the buffer (nullptr: no fused sum)
  unsigned long long* mc;   // multicast address, or nullptr (then peers)
  unsigned long long* peers[TC_MAX_PEERS];
  int world;
  unsigned long long epoch;
  unsigned long long timeout_ns;  // arrival bound (kArrivalTimeoutNs; TC_FUSED_TIMEOUT_MS overrides)
};

__device__ __forceinline__ void fused_sum(unsigned long long* total, const FuseArgs& f) {
  const unsigned long long partial = *(volatile unsigned long long*)total;
  unsigned long long* own = f.own;
  const int slot = (int)(f.epoch & 1ull);
  asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(own + (slot ^ 1)), "l"(0ull) : "memory");
  asm volatile("fence.acq_rel.sys;" ::: "memory");
  if (f.mc) {
    asm volatile("multimem.red.relaxed.sys.global.add.u64 [%0], %1;" ::"l"(f.mc + slot), "l"(partial)
                 : "memory");
    asm volatile("fence.acq_rel.sys;" ::: "memory");
    asm volatile("multimem.red.release.sys.global.add.u64 [%0], %1;" ::"l"(f.mc + 2), "l"(1ull)
                 : "memory");
  } else {
    for (int r = 0; r < f.world; ++r)
      asm volatile("red.relaxed.sys.global.add.u64 [%0], %1;" ::"l"(f.peers[r] + slot), "l"(partial)
                   : "memory");
    asm volatile("fence.acq_rel.sys;" ::: "memory");
    for (int r = 0; r < f.world; ++r)
      asm volatile("red.release.sys.global.add.u64 [%0], %1;" ::"l"(f.peers[r] + 2), "l"(1ull)
                   : "memory");
  }
  const unsigned long long want = (unsigned long long)f.world * f.epoch;
  unsigned long long seen = 0, t0, now;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (;;) {
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(seen) : "l"(own + 2) : "memory");
    if (seen >= want) break;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(now));
    if (now - t0 > f.timeout_ns) {  // a rank never arrived: poison, report, do not hang
      asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(own + 3), "l"(1ull) : "memory");
      *(volatile unsigned long long*)total = ~0ull;
      return;
    }
    __nanosleep(256);
  }
  unsigned long long t;
  asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(t) : "l"(own + slot) : "memory");
  *(volatile unsigned long long*)total = t;
}

// Grid-completion epilogue of a count kernel: called by ONE thread per CTA
// after that CTA's atomicAdd into *total.  The last CTA to finish (ticket in
// word[4] of the own buffer, reset for the next launch) runs fused_sum.
__device__ __forceinline__ void fused_epilogue(unsigned long long* total, const FuseArgs& f) {
  __threadfence();
  const unsigned long long t = atomicAdd(f.own + 4, 1ull);
  if (t + 1 != (unsigned long long)gridDim.x) return;
  __threadfence();
  f.own[4] = 0;  // next launch (stream-ordered after this one)
  fused_sum(total, f);
}

}  // namespace tc

// tc_fused.cu — SURVEY.md §8(f) row f4: the cross-GPU sum of the partial
// counts done by the library itself over NVLink peer memory, instead of an
// NCCL all_reduce.
//
// T = sum over ranks of the partial counts of their edge ranges (the
// per-edge intersections are independent).  After the count kernels of this
// rank's range (tc_count_range's a7/a8/a9), ONE thread of a finishing kernel
//   1. zeroes this rank's replica of the OTHER epoch's sum word,
//   2. adds its partial to the sum word of this epoch on every rank:
//        multicast: one `multimem.red.add.u64` through the NVLS multicast
//                   address (the NVSwitch adds it into every replica), or
//        peers:     one `red.add.u64` per peer replica (P2P over NVLink),
//   3. bumps the arrival word on every rank the same way, with release
//      semantics (so the sum add is visible first),
//   4. spins (acquire) until its own arrival word reaches world * epoch, and
//   5. reads T from its own replica.
// Buffer (symmetric: same layout on every rank, zero-initialised):
//   u64 word[0], word[1] = sum of epochs with parity 0 / 1, word[2] = arrivals.
// The epoch-parity double buffer is safe: rank r clears its replica of slot
// (e+1)&1 before it arrives in epoch e, and no rank adds into that slot (in
// epoch e+1) before it has seen every arrival of epoch e.
#include <cuda.h>

#include <cstring>

#include "tc_internal.cuh"

namespace tc {
namespace {

constexpr unsigned long long kArrivalTimeoutNs = 20ull * 1000 * 1000 * 1000;  // 20 s

struct Peers {
  unsigned long long* p[TC_MAX_PEERS];
};

__global__ void k_fused_finish(unsigned long long* __restrict__ total, unsigned long long* own,
                               unsigned long long* mc, Peers peers, int world,
                               unsigned long long epoch) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  const unsigned long long partial = *total;
  const int slot = (int)(epoch & 1ull);
  // 1. this rank's replica of the other epoch's sum word
  asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(own + (slot ^ 1)), "l"(0ull) : "memory");
  asm volatile("fence.acq_rel.sys;" ::: "memory");
  // 2. + 3. the partial into every replica, then the arrival (release)
  if (mc) {
    asm volatile("multimem.red.relaxed.sys.global.add.u64 [%0], %1;" ::"l"(mc + slot), "l"(partial)
                 : "memory");
    asm volatile("fence.acq_rel.sys;" ::: "memory");
    asm volatile("multimem.red.release.sys.global.add.u64 [%0], %1;" ::"l"(mc + 2), "l"(1ull)
                 : "memory");
  } else {
    for (int r = 0; r < world; ++r)
      asm volatile("red.relaxed.sys.global.add.u64 [%0], %1;" ::"l"(peers.p[r] + slot), "l"(partial)
                   : "memory");
    asm volatile("fence.acq_rel.sys;" ::: "memory");
    for (int r = 0; r < world; ++r)
      asm volatile("red.release.sys.global.add.u64 [%0], %1;" ::"l"(peers.p[r] + 2), "l"(1ull)
                   : "memory");
  }
  // 4. every rank's contribution of this epoch has landed in our replica
  const unsigned long long want = (unsigned long long)world * epoch;
  unsigned long long seen = 0, t0, now;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (;;) {
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(seen) : "l"(own + 2) : "memory");
    if (seen >= want) break;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(now));
    if (now - t0 > kArrivalTimeoutNs) {  // a rank never arrived: report, do not hang
      *total = ~0ull;
      return;
    }
    __nanosleep(256);
  }
  // 5. T
  unsigned long long t;
  asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(t) : "l"(own + slot) : "memory");
  *total = t;
}

// ---------------------------------------------------------------- driver API
// Entry points fetched through the runtime (libtc.so does not link libcuda,
// so it still loads on a machine without a driver for the CPU tests).
template <class F>
F driver_fn(const char* name) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess ||
      q != cudaDriverEntryPointSuccess || !p) {
    cudaGetLastError();
    fail(TC_ERR_UNSUPPORTED, std::string("driver entry point unavailable: ") + name);
  }
  return reinterpret_cast<F>(p);
}

void cu_check(CUresult r, const char* what) {
  if (r != CUDA_SUCCESS)
    fail(r == CUDA_ERROR_NOT_SUPPORTED ? TC_ERR_UNSUPPORTED : TC_ERR_CUDA,
         std::string(what) + " failed (CUresult " + std::to_string((int)r) + ")");
}

}  // namespace

void fused_finish(unsigned long long* d_total, uint64_t* own, uint64_t* mc,
                  uint64_t* const* peers, int world, uint64_t epoch, cudaStream_t s) {
  Peers pp;
  std::memset(&pp, 0, sizeof(pp));
  if (!mc)
    for (int r = 0; r < world; ++r) pp.p[r] = reinterpret_cast<unsigned long long*>(peers[r]);
  k_fused_finish<<<1, 32, 0, s>>>(d_total, reinterpret_cast<unsigned long long*>(own),
                                  reinterpret_cast<unsigned long long*>(mc), pp, world,
                                  (unsigned long long)epoch);
  TC_LAUNCH();
}

void mc_destroy(void* h);

// One process, one device: a multicast object with the current device as its
// only member, its physical memory mapped twice (unicast + multicast VA).
struct McBuffer {
  CUmemGenericAllocationHandle mem = 0, mc = 0;
  CUdeviceptr uc_va = 0, mc_va = 0;
  size_t size = 0;
  int dev = 0;
};

void* mc_create(size_t bytes, uint64_t** uc, uint64_t** mcp) {
  using FnGran = CUresult (*)(size_t*, const CUmulticastObjectProp*, CUmulticastGranularity_flags);
  using FnCreate = CUresult (*)(CUmemGenericAllocationHandle*, const CUmulticastObjectProp*);
  using FnAdd = CUresult (*)(CUmemGenericAllocationHandle, CUdevice);
  using FnMemCreate = CUresult (*)(CUmemGenericAllocationHandle*, size_t, const CUmemAllocationProp*,
                                   unsigned long long);
  using FnBind = CUresult (*)(CUmemGenericAllocationHandle, size_t, CUmemGenericAllocationHandle,
                              size_t, size_t, unsigned long long);
  using FnReserve = CUresult (*)(CUdeviceptr*, size_t, size_t, CUdeviceptr, unsigned long long);
  using FnMap = CUresult (*)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle,
                             unsigned long long);
  using FnAccess = CUresult (*)(CUdeviceptr, size_t, const CUmemAccessDesc*, size_t);
  using FnDevGet = CUresult (*)(CUdevice*, int);
  using FnAttr = CUresult (*)(int*, CUdevice_attribute, CUdevice);
  int ordinal = 0;
  TC_CUDA(cudaGetDevice(&ordinal));
  TC_CUDA(cudaFree(nullptr));  // make sure the primary context exists
  CUdevice dev = 0;
  cu_check(driver_fn<FnDevGet>("cuDeviceGet")(&dev, ordinal), "cuDeviceGet");
  int supported = 0;
  cu_check(driver_fn<FnAttr>("cuDeviceGetAttribute")(&supported,
                                                     CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev),
           "cuDeviceGetAttribute");
  if (!supported) fail(TC_ERR_UNSUPPORTED, "device does not support multicast objects");

  McBuffer* b = new McBuffer();
  b->dev = ordinal;
  try {
  // The driver wants a shareable handle type on the multicast object (and the
  // bound memory) even when it is never exported; try POSIX fd, then fabric.
  const CUmemAllocationHandleType kinds[2] = {CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR,
                                              CU_MEM_HANDLE_TYPE_FABRIC};
  size_t gran = 0;
  CUresult r = CUDA_ERROR_NOT_SUPPORTED;
  CUmemAllocationHandleType kind = kinds[0];
  for (CUmemAllocationHandleType k : kinds) {
    CUmulticastObjectProp mp;
    std::memset(&mp, 0, sizeof(mp));
    mp.numDevices = 1;
    mp.size = bytes;
    mp.handleTypes = (unsigned long long)k;
    r = driver_fn<FnGran>("cuMulticastGetGranularity")(&gran, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED);
    if (r != CUDA_SUCCESS) continue;
    b->size = (bytes + gran - 1) / gran * gran;
    mp.size = b->size;
    r = driver_fn<FnCreate>("cuMulticastCreate")(&b->mc, &mp);
    if (r == CUDA_SUCCESS) {
      kind = k;
      break;
    }
  }
  if (r == CUDA_ERROR_INVALID_VALUE || r == CUDA_ERROR_NOT_PERMITTED || r == CUDA_ERROR_NOT_SUPPORTED)
    // seen on a one-GPU container whose process has no NVSwitch fabric access
    // (every handle type / device count refused, MULTICAST_SUPPORTED = 1)
    fail(TC_ERR_UNSUPPORTED, "cuMulticastCreate refused (CUresult " + std::to_string((int)r) +
                                 "): no NVLS multicast for this process");
  cu_check(r, "cuMulticastCreate");
  cu_check(driver_fn<FnAdd>("cuMulticastAddDevice")(b->mc, dev), "cuMulticastAddDevice");
  CUmemAllocationProp ap;
  std::memset(&ap, 0, sizeof(ap));
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = ordinal;
  ap.requestedHandleTypes = kind;
  cu_check(driver_fn<FnMemCreate>("cuMemCreate")(&b->mem, b->size, &ap, 0), "cuMemCreate");
  cu_check(driver_fn<FnBind>("cuMulticastBindMem")(b->mc, 0, b->mem, 0, b->size, 0),
           "cuMulticastBindMem");
  CUmemAccessDesc acc;
  std::memset(&acc, 0, sizeof(acc));
  acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  acc.location.id = ordinal;
  acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  auto reserve = driver_fn<FnReserve>("cuMemAddressReserve");
  auto map = driver_fn<FnMap>("cuMemMap");
  auto access = driver_fn<FnAccess>("cuMemSetAccess");
  cu_check(reserve(&b->uc_va, b->size, gran, 0, 0), "cuMemAddressReserve");
  cu_check(map(b->uc_va, b->size, 0, b->mem, 0), "cuMemMap (unicast)");
  cu_check(access(b->uc_va, b->size, &acc, 1), "cuMemSetAccess (unicast)");
  cu_check(reserve(&b->mc_va, b->size, gran, 0, 0), "cuMemAddressReserve");
  cu_check(map(b->mc_va, b->size, 0, b->mc, 0), "cuMemMap (multicast)");
  cu_check(access(b->mc_va, b->size, &acc, 1), "cuMemSetAccess (multicast)");
  TC_CUDA(cudaMemset(reinterpret_cast<void*>(b->uc_va), 0, b->size));
  TC_CUDA(cudaDeviceSynchronize());
  } catch (...) {
    mc_destroy(b);
    throw;
  }
  *uc = reinterpret_cast<uint64_t*>(b->uc_va);
  *mcp = reinterpret_cast<uint64_t*>(b->mc_va);
  return b;
}

void mc_destroy(void* h) {
  if (!h) return;
  McBuffer* b = static_cast<McBuffer*>(h);
  using FnUnmap = CUresult (*)(CUdeviceptr, size_t);
  using FnFreeVA = CUresult (*)(CUdeviceptr, size_t);
  using FnRelease = CUresult (*)(CUmemGenericAllocationHandle);
  using FnUnbind = CUresult (*)(CUmemGenericAllocationHandle, CUdevice, size_t, size_t);
  cudaDeviceSynchronize();
  try {
    auto unmap = driver_fn<FnUnmap>("cuMemUnmap");
    auto freeva = driver_fn<FnFreeVA>("cuMemAddressFree");
    auto release = driver_fn<FnRelease>("cuMemRelease");
    auto unbind = driver_fn<FnUnbind>("cuMulticastUnbind");
    if (b->mc_va) { unmap(b->mc_va, b->size); freeva(b->mc_va, b->size); }
    if (b->uc_va) { unmap(b->uc_va, b->size); freeva(b->uc_va, b->size); }
    if (b->mc) { unbind(b->mc, (CUdevice)b->dev, 0, b->size); release(b->mc); }
    if (b->mem) release(b->mem);
  } catch (...) {
  }
  delete b;
}

}  // namespace tc

// tc_fused.cu — SURVEY.md §8(f) row f4: the cross-GPU sum of the partial
// counts done by the library itself over NVLink peer memory, instead of an
// NCCL all_reduce.  The protocol is fused_sum (tc_fused.cuh); normally the
// count kernel's last CTA runs it (tc_count.cu, fused_epilogue), so a fused
// count is the count launches alone.  This file holds the stand-alone
// finishing kernel for a rank whose range launches no count kernel, and the
// single-process multicast buffer (tc_mc_buffer_create).
#include <cuda.h>

#include <cstdlib>
#include <cstring>

#include "tc_fused.cuh"
#include "tc_internal.cuh"

namespace tc {
namespace {

__global__ void k_fused_finish(unsigned long long* __restrict__ total, FuseArgs f) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  fused_sum(total, f);
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

FuseArgs fuse_args(uint64_t* own, uint64_t* mc, uint64_t* const* peers, int world,
                   uint64_t epoch) {
  FuseArgs f;
  std::memset(&f, 0, sizeof(f));
  f.own = reinterpret_cast<unsigned long long*>(own);
  f.mc = reinterpret_cast<unsigned long long*>(mc);
  if (!mc)
    for (int r = 0; r < world; ++r) f.peers[r] = reinterpret_cast<unsigned long long*>(peers[r]);
  f.world = world;
  f.epoch = (unsigned long long)epoch;
  f.timeout_ns = kArrivalTimeoutNs;
  if (const char* e = std::getenv("TC_FUSED_TIMEOUT_MS")) {
    const long long ms = std::atoll(e);
    if (ms > 0) f.timeout_ns = (unsigned long long)ms * 1000000ull;
  }
  return f;
}

void fused_finish(unsigned long long* d_total, const FuseArgs& f, cudaStream_t s) {
  k_fused_finish<<<1, 32, 0, s>>>(d_total, f);
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

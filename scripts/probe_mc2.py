"""Probe cuMulticastCreate parameter combinations on this box (f4)."""
from cuda.bindings import driver as cu

cu.cuInit(0)
_, dev = cu.cuDeviceGet(0)
_, ctx = cu.cuDevicePrimaryCtxRetain(dev)
cu.cuCtxSetCurrent(ctx)
H = cu.CUmemAllocationHandleType
for nd in (1, 2):
    for ht in (H.CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, H.CU_MEM_HANDLE_TYPE_FABRIC, 0):
        for gflag in (cu.CUmulticastGranularity_flags.CU_MULTICAST_GRANULARITY_MINIMUM,
                      cu.CUmulticastGranularity_flags.CU_MULTICAST_GRANULARITY_RECOMMENDED):
            p = cu.CUmulticastObjectProp()
            p.numDevices = nd
            p.handleTypes = int(ht)
            p.size = 2 << 20
            e, g = cu.cuMulticastGetGranularity(p, gflag)
            if e != cu.CUresult.CUDA_SUCCESS:
                print(nd, ht, gflag, "gran", e)
                continue
            p.size = max(g, 2 << 20)
            e2, h = cu.cuMulticastCreate(p)
            print(f"numDevices={nd} handle={ht} gran({gflag})={g} size={p.size} create={e2}")
            if e2 == cu.CUresult.CUDA_SUCCESS:
                e3, = cu.cuMulticastAddDevice(h, dev)
                print("   add device:", e3)
                cu.cuMemRelease(h)

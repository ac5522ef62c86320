"""Probe: does this box expose NVLS multicast to one process (f4 feasibility)?"""
import os
import torch
import torch.distributed as dist

os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
os.environ.setdefault("MASTER_PORT", "29555")
try:
    from cuda.bindings import driver as cu
    cu.cuInit(0)
    err, dev = cu.cuDeviceGet(0)
    err, v = cu.cuDeviceGetAttribute(cu.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev)
    print("CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED", err, v)
    err, v = cu.cuDeviceGetAttribute(cu.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED, dev)
    print("FABRIC_SUPPORTED", err, v)
except Exception as e:
    print("cuda-python probe failed", repr(e))
dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
try:
    import torch.distributed._symmetric_memory as symm
    t = symm.empty(16, dtype=torch.int64, device="cuda")
    h = symm.rendezvous(t, dist.group.WORLD)
    print("symm mem: multicast_ptr", h.multicast_ptr, "buffer_ptrs", h.buffer_ptrs,
          "signal_pad_ptrs", h.signal_pad_ptrs)
except Exception as e:
    print("symm mem failed", repr(e))
dist.destroy_process_group()

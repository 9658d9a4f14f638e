"""Does this box support NVLS multicast objects with the visible GPU(s)?
Prints the device attribute and tries torch symmetric memory (world size 1)."""
import os
import socket

import torch
import torch.distributed as dist

torch.cuda.set_device(0)
from cuda.bindings import driver as d  # noqa: E402

d.cuInit(0)
err, dev = d.cuDeviceGet(0)
err, mc = d.cuDeviceGetAttribute(d.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev)
print("CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED", err, mc, "devices", torch.cuda.device_count())
prop = d.CUmulticastObjectProp()
prop.numDevices = 1
prop.size = 2 << 20
prop.handleTypes = d.CUmemAllocationHandleType.CU_MEM_HANDLE_TYPE_NONE
err, gran = d.cuMulticastGetGranularity(prop, d.CUmulticastGranularity_flags.CU_MULTICAST_GRANULARITY_RECOMMENDED)
print("granularity", err, gran)
err, handle = d.cuMulticastCreate(prop)
print("cuMulticastCreate(1 device, no handle type)", err)
for ht in ("CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR", "CU_MEM_HANDLE_TYPE_FABRIC"):
    prop.handleTypes = getattr(d.CUmemAllocationHandleType, ht)
    err, handle = d.cuMulticastCreate(prop)
    print("cuMulticastCreate(1 device,", ht, ")", err)
    if err == d.CUresult.CUDA_SUCCESS:
        break
if err == d.CUresult.CUDA_SUCCESS:
    print("cuMulticastAddDevice", d.cuMulticastAddDevice(handle, dev)[0])
s = socket.socket()
s.bind(("127.0.0.1", 0))
os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(s.getsockname()[1]))
s.close()
dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
try:
    import torch.distributed._symmetric_memory as symm
    t = symm.empty((1024, 128), dtype=torch.float32, device="cuda")
    h = symm.rendezvous(t, dist.group.WORLD)
    print("symm mem: multicast_ptr", hex(getattr(h, "multicast_ptr", 0) or 0), "buffer_ptrs", h.buffer_ptrs)
except Exception as e:
    print("symm mem failed:", type(e).__name__, e)
dist.destroy_process_group()

# Probe: can this box create a CUDA multicast object (NVLS) for one device?  (gpurun r02nv: no —
# cuMulticastCreate returns INVALID_VALUE for every handle type; tests/test_nvls_gpu.py then skips)
from cuda.bindings import driver as cu
import torch
torch.cuda.init(); torch.zeros(1, device='cuda')
print(cu.cuInit(0))
err, dev = cu.cuDeviceGet(0)
print("mc supported", cu.cuDeviceGetAttribute(cu.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev))
for ht in (cu.CUmemAllocationHandleType.CU_MEM_HANDLE_TYPE_NONE, cu.CUmemAllocationHandleType.CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, cu.CUmemAllocationHandleType.CU_MEM_HANDLE_TYPE_FABRIC):
    p = cu.CUmulticastObjectProp(); p.numDevices = 1; p.handleTypes = ht; p.size = 2 << 20
    print(ht, cu.cuMulticastGetGranularity(p, cu.CUmulticastGranularity_flags.CU_MULTICAST_GRANULARITY_RECOMMENDED))
    r = cu.cuMulticastCreate(p); print("create", r)

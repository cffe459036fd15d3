from cuda.bindings import driver as d
import torch
torch.zeros(1, device="cuda")
for ht in (d.CUmemAllocationHandleType.CU_MEM_HANDLE_TYPE_NONE, d.CUmemAllocationHandleType.CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, d.CUmemAllocationHandleType.CU_MEM_HANDLE_TYPE_FABRIC):
    prop = d.CUmulticastObjectProp()
    prop.numDevices = 1
    prop.size = 2 << 20
    prop.handleTypes = ht
    prop.flags = 0
    err, h = d.cuMulticastCreate(prop)
    print(ht, "create", err)
    if err == d.CUresult.CUDA_SUCCESS:
        print(" add", d.cuMulticastAddDevice(h, 0))

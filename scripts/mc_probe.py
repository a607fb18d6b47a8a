"""Probe: NVLS multicast support on this box (device attribute + a 1-member multicast object)."""
from cuda.bindings import driver as cu
def ck(r):
    if isinstance(r, tuple):
        err, *rest = r
    else:
        err, rest = r, []
    if err != cu.CUresult.CUDA_SUCCESS:
        raise RuntimeError(str(err))
    return rest[0] if len(rest) == 1 else rest
ck(cu.cuInit(0))
dev = ck(cu.cuDeviceGet(0))
print("multicast supported:", ck(cu.cuDeviceGetAttribute(cu.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev)))
ctx = ck(cu.cuDevicePrimaryCtxRetain(dev)); ck(cu.cuCtxSetCurrent(ctx))
prop = cu.CUmulticastObjectProp()
prop.numDevices = 1
prop.size = 2 << 20
prop.handleTypes = cu.CUmemAllocationHandleType.CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR
try:
    gran = ck(cu.cuMulticastGetGranularity(prop, cu.CUmulticastGranularity_flags.CU_MULTICAST_GRANULARITY_RECOMMENDED))
    print("granularity", gran)
    prop.size = max(prop.size, gran)
    mc = ck(cu.cuMulticastCreate(prop))
    ck(cu.cuMulticastAddDevice(mc, dev))
    print("multicast object created with 1 device")
except Exception as e:
    print("multicast create failed:", e)

"""Probe: does this box's B200 support multicast objects (NVLS), and can a 1-device multicast object be
created, bound and mapped, and does multimem.red reach the bound memory?  (Decides whether the
NVLS-fused failed count can be tested on one GPU.)"""
from cuda.bindings import driver as cu


def ck(r):
    err = r[0] if isinstance(r, tuple) else r
    if err != cu.CUresult.CUDA_SUCCESS:
        raise RuntimeError(str(err))
    return r[1:] if isinstance(r, tuple) and len(r) > 1 else None


ck(cu.cuInit(0))
dev, = ck(cu.cuDeviceGet(0))
mc, = ck(cu.cuDeviceGetAttribute(cu.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev))
print("MULTICAST_SUPPORTED", mc)
ctx, = ck(cu.cuDevicePrimaryCtxRetain(dev))
ck(cu.cuCtxSetCurrent(ctx))
HT = cu.CUmemAllocationHandleType
for name in ["CU_MEM_HANDLE_TYPE_NONE", "CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR", "CU_MEM_HANDLE_TYPE_FABRIC"]:
    if not hasattr(HT, name):
        continue
    prop = cu.CUmulticastObjectProp()
    prop.numDevices = 1
    prop.size = 2 << 20
    prop.handleTypes = getattr(HT, name)
    prop.flags = 0
    try:
        mobj, = ck(cu.cuMulticastCreate(prop))
        print(name, "cuMulticastCreate ok")
        ck(cu.cuMulticastAddDevice(mobj, dev))
        print(name, "AddDevice ok")
    except Exception as e:
        print(name, "failed:", e)

"""Probe which multicast-object properties this box's driver accepts (cuda-python)."""
from cuda.bindings import driver as d

def ck(r):
    return r[0] if isinstance(r, tuple) else r

print("init", ck(d.cuInit(0)))
err, dev = d.cuDeviceGet(0)
err, ctx = d.cuDevicePrimaryCtxRetain(dev)
print("ctx", err, d.cuCtxSetCurrent(ctx))
for attr in ("CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED", "CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED",
             "CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR_SUPPORTED"):
    if hasattr(d.CUdevice_attribute, attr):
        print(attr, d.cuDeviceGetAttribute(getattr(d.CUdevice_attribute, attr), dev))
for ht_name in ("CU_MEM_HANDLE_TYPE_NONE", "CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR", "CU_MEM_HANDLE_TYPE_FABRIC"):
    ht = getattr(d.CUmemAllocationHandleType, ht_name)
    for nd in (1, 2):
        for size in (2 << 20, 512 << 20):
            p = d.CUmulticastObjectProp()
            p.numDevices = nd
            p.size = size
            p.handleTypes = int(ht)
            p.flags = 0
            e1, g = d.cuMulticastGetGranularity(p, d.CUmulticastGranularity_flags.CU_MULTICAST_GRANULARITY_MINIMUM)
            e2, g2 = d.cuMulticastGetGranularity(p, d.CUmulticastGranularity_flags.CU_MULTICAST_GRANULARITY_RECOMMENDED)
            e3, h = d.cuMulticastCreate(p)
            print(ht_name, "numDevices", nd, "size", size, "gran", e1, g, e2, g2, "create", e3)
            if e3 == d.CUresult.CUDA_SUCCESS:
                print("   addDevice", d.cuMulticastAddDevice(h, dev))
                d.cuMemRelease(h)

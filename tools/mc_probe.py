# probe: can this box create a CUDA multicast object (NVLS)?  Prints the result per variant.
from cuda.bindings import driver as d
print(d.cuInit(0))
err, dev = d.cuDeviceGet(0)
err, ctx = d.cuDevicePrimaryCtxRetain(dev)
print(d.cuCtxSetCurrent(ctx))
for nd in (1, 2):
    for ht in (0, d.CUmemAllocationHandleType.CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR,
               d.CUmemAllocationHandleType.CU_MEM_HANDLE_TYPE_FABRIC):
        p = d.CUmulticastObjectProp()
        p.numDevices = nd
        p.handleTypes = int(ht)
        p.size = 2 << 20
        e, g = d.cuMulticastGetGranularity(p, d.CUmulticastGranularity_flags.CU_MULTICAST_GRANULARITY_RECOMMENDED)
        p.size = max(g, 2 << 20) if e == 0 else 2 << 20
        r = d.cuMulticastCreate(p)
        print("numDevices", nd, "handleTypes", int(ht), "gran", e, g, "->", r[0])
        if r[0] == 0:
            print("  addDevice", d.cuMulticastAddDevice(r[1], dev))

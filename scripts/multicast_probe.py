"""Probe: are NVLink multicast objects (NVLS, cuMulticastCreate) available on this box's GPU?
Creates a 1-device multicast object, binds 2 MB of device memory, maps the multicast address and
reports each step (used to decide whether NEXT f2 can be exercised on a one-GPU lease)."""
import cuda.bindings.driver as d
d.cuInit(0)
_, dev = d.cuDeviceGet(0)
print("multicast supported attr:", d.cuDeviceGetAttribute(d.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev))
_, ctx = d.cuDevicePrimaryCtxRetain(dev)
d.cuCtxSetCurrent(ctx)
H = d.CUmemAllocationHandleType
for ht in (H.CU_MEM_HANDLE_TYPE_NONE, H.CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, H.CU_MEM_HANDLE_TYPE_FABRIC):
    prop = d.CUmulticastObjectProp()
    prop.numDevices = 1
    prop.size = 2 << 20
    prop.handleTypes = ht
    prop.flags = 0
    r = d.cuMulticastCreate(prop)
    print(ht, "create:", r[0])
    if r[0] != d.CUresult.CUDA_SUCCESS:
        continue
    mc = r[1]
    print("  add device:", d.cuMulticastAddDevice(mc, dev))
    ap = d.CUmemAllocationProp()
    ap.type = d.CUmemAllocationType.CU_MEM_ALLOCATION_TYPE_PINNED
    ap.location.type = d.CUmemLocationType.CU_MEM_LOCATION_TYPE_DEVICE
    ap.location.id = 0
    ap.requestedHandleTypes = ht
    e, mem = d.cuMemCreate(2 << 20, ap, 0)
    print("  mem create:", e)
    print("  bind:", d.cuMulticastBindMem(mc, 0, mem, 0, 2 << 20, 0))
    e, va = d.cuMemAddressReserve(2 << 20, 2 << 20, 0, 0)
    print("  map:", d.cuMemMap(va, 2 << 20, 0, mc, 0))
    acc = d.CUmemAccessDesc()
    acc.location.type = d.CUmemLocationType.CU_MEM_LOCATION_TYPE_DEVICE
    acc.location.id = 0
    acc.flags = d.CUmemAccess_flags.CU_MEM_ACCESS_FLAGS_PROT_READWRITE
    print("  access:", d.cuMemSetAccess(va, 2 << 20, [acc], 1))
    break

"""Probe: does this box support NVLink SHARP multicast objects (f3 prerequisite)?
Prints the device attributes and tries a 1-device multicast object (create, add device,
bind 2 MiB, map)."""
import json

import cuda.bindings.driver as d


def ck(r):
    err = r[0] if isinstance(r, tuple) else r
    if err != d.CUresult.CUDA_SUCCESS:
        raise RuntimeError(str(err))
    return r[1:] if isinstance(r, tuple) and len(r) > 2 else (r[1] if isinstance(r, tuple) and len(r) == 2 else None)


out = {}
ck(d.cuInit(0))
dev = ck(d.cuDeviceGet(0))
ctx = ck(d.cuDevicePrimaryCtxRetain(dev))
ck(d.cuCtxSetCurrent(ctx))
for a in ("CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED", "CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED"):
    out[a] = ck(d.cuDeviceGetAttribute(getattr(d.CUdevice_attribute, a), dev))
try:
    prop = d.CUmulticastObjectProp()
    prop.numDevices = 1
    prop.size = 2 << 20
    prop.handleTypes = d.CUmemAllocationHandleType.CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR
    g = ck(d.cuMulticastGetGranularity(prop, d.CUmulticastGranularity_flags.CU_MULTICAST_GRANULARITY_RECOMMENDED))
    out["granularity"] = int(g)
    mc = ck(d.cuMulticastCreate(prop))
    ck(d.cuMulticastAddDevice(mc, dev))
    ap = d.CUmemAllocationProp()
    ap.type = d.CUmemAllocationType.CU_MEM_ALLOCATION_TYPE_PINNED
    ap.location.type = d.CUmemLocationType.CU_MEM_LOCATION_TYPE_DEVICE
    ap.location.id = 0
    mem = ck(d.cuMemCreate(2 << 20, ap, 0))
    ck(d.cuMulticastBindMem(mc, 0, mem, 0, 2 << 20, 0))
    va = ck(d.cuMemAddressReserve(2 << 20, 2 << 20, 0, 0))
    ck(d.cuMemMap(va, 2 << 20, 0, mc, 0))
    out["multicast_1dev"] = "ok"
except Exception as e:  # noqa: BLE001
    out["multicast_1dev"] = f"failed: {e}"
print(json.dumps(out))

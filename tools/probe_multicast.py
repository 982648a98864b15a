"""Probe NVSwitch multicast on the visible GPUs (CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED and a
one-device cuMulticastCreate + bind + map), as a gate for a multimem.st exchange variant.
Prints one JSON line."""
import ctypes
import json


def main():
    cu = ctypes.CDLL("libcuda.so.1")
    out = {}
    rc = cu.cuInit(0)
    n = ctypes.c_int()
    cu.cuDeviceGetCount(ctypes.byref(n))
    out["devices"] = n.value
    devs = []
    for d in range(n.value):
        dev = ctypes.c_int()
        cu.cuDeviceGet(ctypes.byref(dev), d)
        mc = ctypes.c_int(-1)
        fab = ctypes.c_int(-1)
        cu.cuDeviceGetAttribute(ctypes.byref(mc), 132, dev)   # MULTICAST_SUPPORTED
        cu.cuDeviceGetAttribute(ctypes.byref(fab), 128, dev)  # HANDLE_TYPE_FABRIC_SUPPORTED
        devs.append({"multicast_supported": mc.value, "fabric_handle_supported": fab.value})
    out["per_device"] = devs
    if n.value and devs[0]["multicast_supported"] == 1:
        # CUmulticastObjectProp {unsigned numDevices; size_t size; unsigned long long handleTypes; unsigned long long flags}
        class Prop(ctypes.Structure):
            _fields_ = [("numDevices", ctypes.c_uint), ("size", ctypes.c_size_t),
                        ("handleTypes", ctypes.c_ulonglong), ("flags", ctypes.c_ulonglong)]
        ctx = ctypes.c_void_p()
        dev = ctypes.c_int()
        cu.cuDeviceGet(ctypes.byref(dev), 0)
        out["ctx_rc"] = cu.cuDevicePrimaryCtxRetain(ctypes.byref(ctx), dev)
        cu.cuCtxSetCurrent(ctx)
        p = Prop(1, 2 << 20, 0, 0)
        gran = ctypes.c_size_t()
        out["gran_rc"] = cu.cuMulticastGetGranularity(ctypes.byref(gran), ctypes.byref(p), 1)
        out["granularity"] = gran.value
        p.size = max(gran.value, 2 << 20)
        h = ctypes.c_ulonglong()
        out["create_rc"] = cu.cuMulticastCreate(ctypes.byref(h), ctypes.byref(p))
        if out["create_rc"] == 0:
            out["add_device_rc"] = cu.cuMulticastAddDevice(h, dev)
    print(json.dumps(out))


if __name__ == "__main__":
    main()

"""cuMulticastCreate over numDevices x handleTypes x size on the visible device (diagnostic
for the multicast exchange: which object properties the driver accepts here)."""
import ctypes
import json


class Prop(ctypes.Structure):
    _fields_ = [("numDevices", ctypes.c_uint), ("size", ctypes.c_size_t),
                ("handleTypes", ctypes.c_ulonglong), ("flags", ctypes.c_ulonglong)]


def main():
    cu = ctypes.CDLL("libcuda.so.1")
    cu.cuInit(0)
    dev = ctypes.c_int()
    cu.cuDeviceGet(ctypes.byref(dev), 0)
    ctx = ctypes.c_void_p()
    cu.cuDevicePrimaryCtxRetain(ctypes.byref(ctx), dev)
    cu.cuCtxSetCurrent(ctx)
    drv = ctypes.c_int()
    cu.cuDriverGetVersion(ctypes.byref(drv))
    out = {"driver": drv.value, "tries": []}
    for nd in (1, 2):
        for ht in (0, 1, 8):
            for size in (2 << 20, 32 << 20, 512 << 20):
                p = Prop(nd, size, ht, 0)
                g = ctypes.c_size_t()
                grc = cu.cuMulticastGetGranularity(ctypes.byref(g), ctypes.byref(p), 0)
                h = ctypes.c_ulonglong()
                rc = cu.cuMulticastCreate(ctypes.byref(h), ctypes.byref(p))
                add = None
                if rc == 0:
                    add = cu.cuMulticastAddDevice(h, dev)
                    cu.cuMemRelease(h)
                out["tries"].append({"numDevices": nd, "handleTypes": ht, "size": size, "gran_rc": grc,
                                     "gran": g.value, "create_rc": rc, "add_rc": add})
    print(json.dumps(out))


if __name__ == "__main__":
    main()

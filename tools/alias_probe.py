#!/usr/bin/env python3
"""Can the device map a full-size host key span backed by fewer physical pages?  Builds
synth.AliasedHostTable spans (one memfd mapped k times) and page-locks + maps them with
cudaHostRegister -- the whole span in one call, or each alias copy in its own call -- and
reports the status, the time, whether the device pointer equals the host pointer (UVA), and
a device read through the last copy."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import numpy as np
    import torch
    import synth
    import ctypes
    torch.cuda.set_device(0)
    torch.zeros(1, device="cuda")
    rt = ctypes.CDLL("libcudart.so.12")      # the runtime torch already loaded
    rt.cudaHostRegister.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_uint]
    rt.cudaHostUnregister.argtypes = [ctypes.c_void_p]
    rt.cudaMemcpy.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int]
    R = 512
    for phys_gb, copies, flags in [(4, 2, 3), (4, 2, 11), (4, 8, 3), (60, 7, 3)]:
        phys = int(phys_gb * 1e9) // R
        t = synth.AliasedHostTable(phys * copies, R, phys)
        t.fill()
        res = {"phys_gb": phys_gb, "copies": copies, "span_gb": t.nbytes / 1e9, "flags": flags}
        t0 = time.time()
        res["whole_span_status"] = int(rt.cudaHostRegister(t.ptr, t.nbytes, flags))
        res["whole_span_s"] = time.time() - t0
        if res["whole_span_status"] == 0:
            rt.cudaHostUnregister(t.ptr)
        rt.cudaGetLastError()
        t0 = time.time()
        sts = []
        for i in range(t.copies):
            sts.append(int(rt.cudaHostRegister(t.ptr + i * t.phys_bytes, t.phys_bytes, flags)))
            rt.cudaGetLastError()
        res["per_copy_status"] = sts
        res["per_copy_s"] = time.time() - t0
        if all(x == 0 for x in sts):
            # UVA: each copy's device address is its host address, so the device sees the
            # whole span; read a row of the last copy through it
            dptrs = []
            for i in range(t.copies):
                d = ctypes.c_void_p()
                rt.cudaHostGetDevicePointer(ctypes.byref(d), ctypes.c_void_p(t.ptr + i * t.phys_bytes), 0)
                dptrs.append(d.value == t.ptr + i * t.phys_bytes)
            res["device_ptr_is_host_ptr"] = all(dptrs)
            k = (t.copies - 1) * t.phys_rows + 12345
            row = torch.empty(R, dtype=torch.uint8, device="cuda")
            rt.cudaMemcpy(ctypes.c_void_p(row.data_ptr()), ctypes.c_void_p(t.ptr + k * R), R, 4)
            torch.cuda.synchronize()
            res["device_read_ok"] = bool(np.array_equal(row.cpu().numpy(),
                                                        synth.rows_for_keys(np.array([12345]), phys, R)[0]))
        for i, x in enumerate(sts):
            if x == 0:
                rt.cudaHostUnregister(t.ptr + i * t.phys_bytes)
        rt.cudaGetLastError()
        print(json.dumps(res), flush=True)
        t.close()


if __name__ == "__main__":
    main()

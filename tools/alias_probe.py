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
    torch.cuda.set_device(0)
    rt = torch.cuda.cudart()
    R = 512
    for phys_gb, copies, flags in [(4, 2, 11), (4, 2, 3), (4, 8, 3), (60, 7, 3)]:
        phys = int(phys_gb * 1e9) // R
        t = synth.AliasedHostTable(phys * copies, R, phys)
        t.fill()
        res = {"phys_gb": phys_gb, "copies": copies, "span_gb": t.nbytes / 1e9, "flags": flags}
        t0 = time.time()
        st = rt.cudaHostRegister(t.ptr, t.nbytes, flags)
        res["whole_span_status"] = int(st.value) if hasattr(st, "value") else int(st)
        res["whole_span_s"] = time.time() - t0
        if res["whole_span_status"] == 0:
            rt.cudaHostUnregister(t.ptr)
        torch.cuda.synchronize()
        t0 = time.time()
        sts = []
        for i in range(t.copies):
            st = rt.cudaHostRegister(t.ptr + i * t.phys_bytes, t.phys_bytes, flags)
            sts.append(int(st.value) if hasattr(st, "value") else int(st))
        res["per_copy_status"] = sts
        res["per_copy_s"] = time.time() - t0
        if all(x == 0 for x in sts):
            # read row k in the last copy through the device: a uint8 tensor view over the
            # host pointer (UVA: device address == host address for registered memory)
            k = (t.copies - 1) * t.phys_rows + 12345
            keys = torch.tensor([k], dtype=torch.int64, device="cuda")
            import ctypes
            base = t.ptr
            buf = (ctypes.c_uint8 * t.nbytes).from_address(base)
            host_view = torch.frombuffer(buf, dtype=torch.uint8)
            row = torch.empty(R, dtype=torch.uint8, device="cuda")
            row.copy_(host_view[k * R:(k + 1) * R], non_blocking=True)
            torch.cuda.synchronize()
            res["device_read_ok"] = bool(np.array_equal(row.cpu().numpy(), synth.rows_for_keys(np.array([12345]), phys, R)[0]))
            for i in range(t.copies):
                rt.cudaHostUnregister(t.ptr + i * t.phys_bytes)
        print(json.dumps(res), flush=True)
        t.close()


if __name__ == "__main__":
    main()

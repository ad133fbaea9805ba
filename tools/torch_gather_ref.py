#!/usr/bin/env python3
"""Reference point for the HBM-bound path: a library gather of the same shape (torch
index_select of 500K random 512-B rows out of a large device slab, CUDA events, distinct index
sets, L2 flushed before each) -- what a vendor gather kernel reaches on random 512-B rows,
next to the single pass (which also locates every key through the location table)."""
import json
import sys

import torch


def main():
    rows = int(sys.argv[1]) if len(sys.argv) > 1 else 16_000_000   # 8.2 GB slab
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 500_000
    R = 512
    dev = torch.device("cuda", 0)
    slab = torch.empty((rows, R // 4), dtype=torch.float32, device=dev)
    slab.view(torch.int32).random_()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    idx = [torch.randint(0, rows, (n,), device=dev) for _ in range(8)]
    out = torch.empty((n, R // 4), dtype=torch.float32, device=dev)
    res = {}
    for mode in ("cold", "steady"):
        ms = []
        for i in range(16):
            if mode == "cold":
                flush.fill_(i & 0xFF)
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            torch.index_select(slab, 0, idx[i % 8], out=out)
            e.record()
            torch.cuda.synchronize()
            if i >= 4:
                ms.append(s.elapsed_time(e))
        t = sorted(ms)[len(ms) // 2]
        res[mode] = {"ms": t, "GBps_rows_read_plus_written": 2 * n * R / (t * 1e-3) / 1e9}
    print(json.dumps({"what": "torch.index_select, random 512-B rows", "slab_rows": rows, "n": n, **res}))


if __name__ == "__main__":
    main()

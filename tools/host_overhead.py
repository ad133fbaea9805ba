#!/usr/bin/env python3
"""Per-call cost of ugache_extract on the host and back to back on the device, by batch size
(small batches are where a fixed cost shows).  gnn_pa@0.25 table, UGache placement, G = 1 or G
fake peers; factored path (auto) vs random dispatch.

  host_us   : wall time per call of UGache.extract (Python binding + C ABI), 500 calls
              enqueued without a sync (the device runs behind; the queue never fills)
  abi_us    : the same through a direct ctypes call with pre-marshalled arguments
  device_us : CUDA-event time per extract over 200 back-to-back extracts (no flush, distinct
              batches cycled), i.e. the steady-state cost per batch including launch gaps
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="gnn_pa@0.25")
    ap.add_argument("--gpus", type=int, nargs="+", default=[1, 4])
    ap.add_argument("--batch-n", type=int, nargs="+", default=[2000, 20000, 100000])
    ap.add_argument("--cache-ratio", type=float, default=0.2)
    args = ap.parse_args()
    import dataclasses
    import torch
    import synth
    from paper_conf_sosp_songz0c23_b200 import (UGache, connect_in_process, fill_host_tier,
                                                host_tier_rows, make_config, solve)
    from paper_conf_sosp_songz0c23_b200 import _abi
    from paper_conf_sosp_songz0c23_b200.ugache import lib
    wl0 = synth.get_workload(args.workload)
    N, R = wl0.num_rows, wl0.row_bytes
    C = int(round(N * args.cache_ratio))
    torch.cuda.set_device(0)
    table = synth.HostTable(N, R)
    table.fill()
    h = synth.hotness(wl0)
    stream = torch.cuda.Stream()
    for G in args.gpus:
        cfg = make_config(N, R, C, num_gpus=G, policy="ugache", host_tier=True)
        plan, order = solve(cfg, h)
        tier = synth.HostTable(host_tier_rows(plan, N), R)
        fill_host_tier(cfg, order, plan, table, tier)
        group = [UGache(table, N, R, C, num_gpus=G, rank=g, device=0, policy="ugache", plan=plan,
                        order=order, host_tier=tier) for g in range(G)]
        connect_in_process(group)
        for cc in group:
            cc.fill()
        torch.cuda.synchronize()
        c = group[0]
        for n in args.batch_n:
            wl = dataclasses.replace(wl0, batch_n=n)
            keys = [torch.from_numpy(synth.make_batch(wl, 0, b)).cuda() for b in range(8)]
            out = torch.empty((n, R), dtype=torch.uint8, device="cuda")
            for mode in ("factored", "random"):
                c.set_mode(mode)
                with torch.cuda.stream(stream):
                    for i in range(20):
                        c.extract(keys[i % 8], out, stream)
                stream.synchronize()
                # host cost per call through the Python binding
                torch.cuda._sleep(2_000_000_000 // 1000)   # ~1 ms of device work ahead of the calls
                t0 = time.perf_counter()
                for i in range(500):
                    c.extract(keys[i % 8], out, stream)
                host_us = (time.perf_counter() - t0) / 500 * 1e6
                stream.synchronize()
                # host cost per call of the bare C ABI
                kp = [k.data_ptr() for k in keys]
                op, sh = out.data_ptr(), stream.cuda_stream
                f = lib().ugache_extract
                t0 = time.perf_counter()
                for i in range(500):
                    f(c.ctx, kp[i % 8], _abi.KEY_I64, n, op, sh)
                abi_us = (time.perf_counter() - t0) / 500 * 1e6
                stream.synchronize()
                # device time per extract, back to back
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                with torch.cuda.stream(stream):
                    torch.cuda._sleep(20_000_000)          # let the host get ahead
                    s.record(stream)
                    for i in range(200):
                        f(c.ctx, kp[i % 8], _abi.KEY_I64, n, op, sh)
                    e.record(stream)
                stream.synchronize()
                dev_us = s.elapsed_time(e) / 200 * 1e3
                r = {"G": G, "n": n, "mode": mode, "path": c.last_extract_path(), "host_us": round(host_us, 2),
                     "abi_us": round(abi_us, 2), "device_us": round(dev_us, 2)}
                print(json.dumps(r), flush=True)
            c.set_mode("factored")
        for cc in group:
            cc.close()
        tier.close()
        del group
        torch.cuda.empty_cache()
    table.close()


if __name__ == "__main__":
    main()

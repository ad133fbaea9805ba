#!/usr/bin/env python3
"""bench.py -- UGache factored embedding extraction on B200 (one process per GPU).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload gnn_pa] [--cache-ratio 0.1]
                  [--policy ugache|replication|partition] [--mode factored|random]
                  [--impl ours|reference]

A step is one ugache_extract of one batch (locate + bucket + factored gather, SURVEY.md
8(a) rows A1-A4) per GPU.  Default workload: BASELINE.json configs[1] (Papers100M-shaped,
111M x 128 fp32 rows = 56.8 GB host table, 500K unique Zipf(1.2) keys per GPU per batch,
10 % per-GPU cache).  Prints ONE JSON line on rank 0.

Timing: W warm-up steps; then K steps back to back on the extract stream (steady state: no
L2 flush -- every step's rows, outputs and location-table lines exceed the 126 MB L2 and the
steps cycle through --batches distinct key sets -- and no per-step host sync), CUDA events
between consecutive steps; barrier + synchronize on both sides; per-rank time = sum of the K
event intervals; value = bytes of all ranks / max over ranks.  `cold_l2`: the same K steps
with a 256 MiB L2-flush write (and a ~50 us spin) before each, outside the events.  e2e: the
same metric through UGache.extract with pinned HOST keys (read in place) and a stats
readback, host wall clock.  --impl reference times the CPU oracle (oracle/gather.c).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "extraction GB/s (n*R/t_batch, all GPUs), ms/batch, % of source-mix roofline"
NVLINK_GBS = 770.0   # B200_PROFILING.md: measured peer copy per direction


def batch_roofline(P, n, R, kb, path, hbm, pcie, nvl):
    """Source-mix roofline of one batch on every GPU.

    P[g, j]: keys GPU g read from source j in the batch (j = g local, j < G peer, j = G host);
    n[g]: keys of GPU g's batch; R: row bytes; kb: key bytes; path: the extract path taken;
    hbm / nvl: GB/s; pcie[g]: GB/s of GPU g's host link.  Per GPU, algorithmic bytes:
      HBM      n_L*R (local reads) + n*R (out writes) + n*(kb + 8) (keys + location entries)
               + bucket traffic (16 B/key two-phase; 16 B per queued peer key single pass)
               + B_served (rows the peers read from this GPU's slab)
      NVLink   ingress sum_j n_Pj*R; egress B_served
      PCIe     n_H*R
    T_roof(g) = max of the four terms / their bandwidths; the batch roofline is max over g.
    Also the bytes of the timed kernel alone ("kernel_bytes": the split path times K2 only,
    whose HBM bytes are n_L*R + n*R + 8n bucket reads + B_served)."""
    P = np.asarray(P, dtype=np.float64)
    G = P.shape[0]
    served = P[:, :G].sum(axis=0) - np.diag(P[:, :G])          # rows read from g by peers
    ranks = []
    for g in range(G):
        n_l, n_h = P[g, g], P[g, G]
        n_p = P[g, :G].sum() - n_l
        bucket = 16.0 * (n_p if path == "single_pass" else n[g])
        b = {"hbm": n_l * R + n[g] * R + n[g] * (kb + 8) + bucket + served[g] * R,
             "pcie": n_h * R, "nvlink_in": n_p * R, "nvlink_out": served[g] * R}
        kbytes = dict(b)
        if path == "split":
            kbytes["hbm"] = n_l * R + n[g] * R + 8.0 * n[g] + served[g] * R
        bw = {"hbm": hbm, "pcie": pcie[g], "nvlink_in": nvl, "nvlink_out": nvl}
        t = {k: (b[k] / (bw[k] * 1e9) if bw[k] else 0.0) for k in b}
        kt = {k: (kbytes[k] / (bw[k] * 1e9) if bw[k] else 0.0) for k in b}
        ranks.append({"bytes": b, "t_s": t, "t_roof_s": max(t.values()), "bound": max(t, key=t.get),
                      "kernel_bytes": kbytes, "kernel_bound": max(kt, key=kt.get)})
    bounding = int(np.argmax([r["t_roof_s"] for r in ranks]))
    return {"ranks": ranks, "t_roof_s": ranks[bounding]["t_roof_s"], "bounding_rank": bounding}


def log(*a):
    print("[bench]", *a, file=sys.stderr, flush=True)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--workload", default="gnn_pa")
    ap.add_argument("--cache-ratio", type=float, default=None)
    ap.add_argument("--alpha", type=float, default=None, help="Zipf alpha (default: the workload's)")
    ap.add_argument("--policy", default="ugache")
    ap.add_argument("--mode", default="factored", choices=["factored", "random"])
    ap.add_argument("--stream", default="auto", choices=["off", "on", "auto"],
                    help="single-pass extraction (UGACHE_OPT_STREAM)")
    ap.add_argument("--inline", default="host", choices=["host", "none", "all"],
                    help="single pass: sources copied by the locating warps (UGACHE_OPT_INLINE)")
    ap.add_argument("--host-sms", type=int, default=0)
    ap.add_argument("--peer-sms", type=int, default=0)
    ap.add_argument("--batches", type=int, default=8, help="distinct batches cycled per rank")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--no-verify", action="store_true")
    ap.add_argument("--no-clocks", action="store_true", help="do not sample nvidia-smi (diagnostics only)")
    ap.add_argument("--host-tier", dest="host_tier", action="store_true", default=True,
                    help="read host rows from a hotness-ordered pinned copy (UGACHE_FLAG_HOST_TIER, "
                         "default)")
    ap.add_argument("--no-host-tier", dest="host_tier", action="store_false")
    ap.add_argument("--extra", dest="extra", action="store_true", default=True,
                    help="also time the random-dispatch (unfactored) ablation (default)")
    ap.add_argument("--no-extra", dest="extra", action="store_false")
    ap.add_argument("--share-gpus", action="store_true",
                    help="allow more ranks than visible GPUs (functional multi-rank runs on one "
                         "GPU; gloo control plane); otherwise that is an error")
    ap.add_argument("--alias-gb", type=float, default=0.0,
                    help="full-size key span on a smaller box: back the N-row host table with this "
                         "many GB of physical rows mapped repeatedly (synth.AliasedHostTable); the "
                         "host tier is then off (it would need the full span physically)")
    ap.add_argument("--calibrate", dest="calibrate", action="store_true", default=True,
                    help="run ugache_calibrate (A0) on every rank at once before timing and report "
                         "the curves in the JSON line (default)")
    ap.add_argument("--no-calibrate", dest="calibrate", action="store_false")
    ap.add_argument("--print-world", action="store_true",
                    help="print this rank's RANK/WORLD_SIZE as JSON and exit (launch check)")
    return ap.parse_args()


def _free_port() -> int:
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def launch_ranks(args):
    """--gpus N (N > 1) needs N ranks, one per GPU.  Under torchrun WORLD_SIZE must equal N
    (else exit 2).  Without a torchrun environment, re-run this very command under
    torch.distributed.run with N local ranks (127.0.0.1 rendezvous) and exit with its status,
    so `python bench.py --gpus N` never silently measures one GPU."""
    ws_env = os.environ.get("WORLD_SIZE")
    if ws_env is not None:
        if int(ws_env) != args.gpus and args.impl != "reference":
            log(f"error: --gpus {args.gpus} but WORLD_SIZE {ws_env}")
            sys.exit(2)
        return
    if args.gpus <= 1 or args.impl == "reference":
        return
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={args.gpus}", "--master-addr", "127.0.0.1",
           "--master-port", str(_free_port()), os.path.abspath(__file__)] + sys.argv[1:]
    log("launching " + " ".join(cmd[1:]))
    sys.exit(subprocess.run(cmd).returncode)


def shm_plan(bytes_needed: int, path: str = "/dev/shm"):
    """(ok, free bytes) of the shared-memory filesystem that holds the node's host table and
    host tier at N > 1."""
    try:
        st = os.statvfs(path)
        free = st.f_bavail * st.f_frsize
    except OSError:
        return False, 0
    return bytes_needed <= free, free


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, ws, local


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, index: int):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return None
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.flush()
        rows = []
        with open(self.f.name) as fh:
            for line in fh:
                parts = [x.strip() for x in line.split(",")]
                if len(parts) >= 9:
                    rows.append(parts)
        os.unlink(self.f.name)
        if not rows:
            return None
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons,
                "samples": len(rows)}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except Exception:
        return {}


def pcie_h2d_peak(torch) -> float:
    """Live PCIe reference: pinned-host -> device cudaMemcpy of 1 GiB, best of 10 (GB/s)."""
    n = 1 << 30
    h = torch.empty(n, dtype=torch.uint8).pin_memory()
    d = torch.empty(n, dtype=torch.uint8, device="cuda")
    best = 1e9
    for _ in range(10):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        d.copy_(h, non_blocking=True)
        e.record()
        torch.cuda.synchronize()
        best = min(best, s.elapsed_time(e))
    del h, d
    return n / (best * 1e-3) / 1e9


def mem_available() -> int:
    try:
        with open("/proc/meminfo") as f:
            for line in f:
                if line.startswith("MemAvailable:"):
                    return int(line.split()[1]) * 1024
    except OSError:
        pass
    return 0


def pin_alias_copies(table):
    """Page-lock an AliasedHostTable copy by copy (the driver refuses one cudaHostRegister
    over a span that maps the same physical pages twice) and check that every copy's device
    address is its host address (UVA), so the library -- which uses already-pinned memory as
    is -- reaches the whole span through the base pointer.  Returns the unpin function."""
    import ctypes
    rt = ctypes.CDLL("libcudart.so.12")
    rt.cudaHostRegister.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_uint]
    rt.cudaHostUnregister.argtypes = [ctypes.c_void_p]
    rt.cudaHostGetDevicePointer.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint]
    done = []
    for i in range(table.copies):
        p = table.ptr + i * table.phys_bytes
        n = min(table.phys_bytes, table.ptr + table.nbytes - p)
        st = rt.cudaHostRegister(p, n, 1 | 2 | 8)          # portable | mapped | read-only
        if st:
            rt.cudaGetLastError()
            st = rt.cudaHostRegister(p, n, 1 | 2)
        if st:
            raise RuntimeError(f"cudaHostRegister of alias copy {i} failed: {st}")
        done.append(p)
        d = ctypes.c_void_p()
        rt.cudaHostGetDevicePointer(ctypes.byref(d), p, 0)
        if d.value != p:
            raise RuntimeError("registered host memory is not identity-mapped (UVA); aliased spans "
                               "cannot be presented to the device as one range")

    def unpin():
        for p in done:
            rt.cudaHostUnregister(p)
    return unpin


def setup_table(wl, rank, ws, torch_dist, alias_gb=0.0):
    import synth
    t0 = time.time()
    if alias_gb > 0 and wl.table_bytes > alias_gb * 1e9:
        if ws > 1:
            raise SystemExit("--alias-gb is single-process only")
        table = synth.AliasedHostTable(wl.num_rows, wl.row_bytes, int(alias_gb * 1e9) // wl.row_bytes)
        table.fill()
        log(f"aliased table: {wl.num_rows} rows x {wl.row_bytes} B span ({wl.table_bytes / 1e9:.1f} GB) "
            f"backed by {table.phys_rows} physical rows ({table.phys_bytes / 1e9:.1f} GB) mapped "
            f"{table.copies} times, in {time.time() - t0:.1f}s")
        return table
    if ws == 1:
        table = synth.HostTable(wl.num_rows, wl.row_bytes)
        table.fill()
    else:
        path = f"/dev/shm/ugache_bench_{wl.name}_{os.environ.get('MASTER_PORT', '0')}"
        if rank == 0:
            table = synth.HostTable(wl.num_rows, wl.row_bytes, shm_path=path, create=True)
            table.fill()
        torch_dist.barrier()
        if rank != 0:
            table = synth.HostTable(wl.num_rows, wl.row_bytes, shm_path=path, create=False)
    log(f"table {wl.num_rows} x {wl.row_bytes} B = {wl.table_bytes / 1e9:.1f} GB ready in "
        f"{time.time() - t0:.1f}s")
    return table


def make_batches(wl, rank, nb):
    """nb distinct seeded batches of this rank (generated in parallel host threads)."""
    import synth
    from concurrent.futures import ThreadPoolExecutor
    t0 = time.time()
    synth.zipf_cdf(wl.table_rows[0], wl.alpha)      # build the shared CDF once
    with ThreadPoolExecutor(max_workers=min(nb, max(1, (os.cpu_count() or 8) // 2))) as ex:
        b = list(ex.map(lambda i: synth.make_batch(wl, rank, i), range(nb)))
    log(f"{nb} batches of {len(b[0])} keys in {time.time() - t0:.1f}s")
    return b


def run_reference(args, wl):
    """--impl reference: the CPU oracle (plain OpenMP gather) on the box's host cores."""
    import oracle
    rank, ws, _ = dist_env()
    if rank != 0:
        return
    import synth
    avail = mem_available()
    if args.alias_gb > 0 and wl.table_bytes > args.alias_gb * 1e9:
        table = setup_table(wl, 0, 1, None, args.alias_gb)
    elif avail and wl.table_bytes > 0.9 * avail:
        print(json.dumps({"impl": "reference", "unavailable": f"the {wl.table_bytes / 1e9:.0f} GB table does "
                          f"not fit host RAM; rerun with --alias-gb"}), flush=True)
        return
    else:
        table = synth.HostTable(wl.num_rows, wl.row_bytes)
        table.fill()
    batches = make_batches(wl, 0, max(1, min(args.batches, args.steps)))
    n = len(batches[0])
    out = np.empty((n, wl.row_bytes), dtype=np.uint8)
    for i in range(args.warmup):
        oracle.gather(table.ptr, wl.num_rows, wl.row_bytes, batches[i % len(batches)], out)
    times = []
    for i in range(args.steps):
        t = time.perf_counter()
        oracle.gather(table.ptr, wl.num_rows, wl.row_bytes, batches[i % len(batches)], out)
        times.append(time.perf_counter() - t)
    tot = sum(times)
    gbs = args.steps * n * wl.row_bytes / tot / 1e9
    cores = len(os.sched_getaffinity(0))
    line = {"metric": METRIC, "value": gbs, "unit": "GB/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": tot / args.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u8",
            "data": "synthetic", "impl": "reference",
            "config": config_dict(args, wl, ws),
            "cpu_baseline": {"value": gbs, "unit": "GB/s", "cores": cores, "kind": "oracle",
                             "sample": f"{args.steps} full batches of {n} keys (oracle/gather.c, "
                                       f"OpenMP, {cores} threads) on rank 0"},
            "e2e": {"value": gbs, "unit": "GB/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def config_dict(args, wl, ws):
    return {"workload": wl.name, "num_rows": wl.num_rows, "row_bytes": wl.row_bytes,
            "payload": f"{wl.row_bytes // (2 if wl.dtype == 'f16' else 4)} x {wl.dtype}",
            "keys_per_batch_per_gpu": wl.keys_per_batch, "batch_kind": wl.batch_kind,
            "alpha": wl.alpha, "cache_ratio": args.cache_ratio if args.cache_ratio is not None
            else wl.cache_ratio, "policy": args.policy, "mode": args.mode, "stream": args.stream, "inline": args.inline,
            "host_tier": bool(getattr(args, "host_tier", False)),
            "host_table": (f"aliased: {args.alias_gb:g} GB of physical rows mapped over the full "
                           f"{wl.table_bytes / 1e9:.0f} GB span" if getattr(args, "alias_gb", 0) and
                           wl.table_bytes > args.alias_gb * 1e9 else "full"),
            "parallelism": f"dp{ws}",
            "l2": "inputs larger than L2: no flush between the back-to-back timed steps; every step "
                  "reads and writes its batch's rows (> 0.25 GB) and touches one location-table line "
                  "per key, against a 126 MB L2, and the steps cycle through distinct key sets "
                  "(--batches); the cold-L2 variant (256 MiB flush before each step) is cold_l2",
            "batches": getattr(args, "batches", None)}


def role_summary(tl, num_gpus, rank):
    """Per-role view of the last fused launch's per-CTA timeline (ugache_last_batch_timeline):
    CTAs per role and median / max of gather start, role done and CTA done, in us from the
    kernel's start -- which source's SMs bound the batch (the paper's Fig. 8 picture)."""
    roles = {}
    for row in tl:
        src = int(row[0])
        name = ("host" if src == num_gpus else "mixed" if src == num_gpus + 1
                else "local" if src == rank else f"peer{src}")
        roles.setdefault(name, []).append(row)
    out = {}
    for name, rows in sorted(roles.items()):
        a = np.array(rows) * 1e3
        out[name] = {"ctas": len(rows),
                     "gather_start": [round(float(np.median(a[:, 2])), 2), round(float(a[:, 2].max()), 2)],
                     "role_done": [round(float(np.median(a[:, 3])), 2), round(float(a[:, 3].max()), 2)],
                     "cta_done": [round(float(np.median(a[:, 4])), 2), round(float(a[:, 4].max()), 2)]}
    out["how"] = ("per-CTA %globaltimer stamps of the last timed fused launch (rank 0): [median, max] "
                  "us from the kernel's start; role_done = the CTA's own source drained, cta_done "
                  "= after local padding")
    return out


def main():
    args = parse()
    launch_ranks(args)
    if args.print_world:
        rank, ws, local = dist_env()
        print(json.dumps({"rank": rank, "world_size": ws, "local_rank": local, "gpus": args.gpus}),
              flush=True)
        return
    import synth
    wl = synth.get_workload(args.workload)
    if args.cache_ratio is not None:
        from dataclasses import replace
        wl = replace(wl, cache_ratio=args.cache_ratio)
    if args.alpha is not None:   # Zipf skew of the keys and hotness (GNN 1.2 plus 1.4)
        from dataclasses import replace
        wl = replace(wl, alpha=args.alpha)
    if args.impl == "reference":
        run_reference(args, wl)
        return

    import torch
    import torch.distributed as tdist
    from paper_conf_sosp_songz0c23_b200 import UGache, dist as ugdist, make_config, solve
    rank, ws, local = dist_env()
    ndev = torch.cuda.device_count()
    if ndev < 1:
        log("error: no CUDA device visible")
        sys.exit(3)
    if ws > ndev and not args.share_gpus:
        log(f"error: {ws} ranks but only {ndev} GPUs visible (use --share-gpus for a functional "
            f"multi-rank run on shared GPUs)")
        sys.exit(3)
    if ws > 1:
        # the node's host table (+ tier) live in /dev/shm, shared by the ranks
        need = wl.table_bytes * (2 if args.host_tier else 1)
        ok, free = shm_plan(need)
        if not ok and args.host_tier and shm_plan(wl.table_bytes)[0]:
            log(f"/dev/shm has {free / 1e9:.1f} GB free < table + tier {need / 1e9:.1f} GB: "
                f"running without the shared host tier")
            args.host_tier = False
        elif not ok:
            log(f"error: /dev/shm has {free / 1e9:.1f} GB free < host table {wl.table_bytes / 1e9:.1f} GB")
            sys.exit(4)
    dev_idx = local % ndev
    torch.cuda.set_device(dev_idx)
    dev = torch.device("cuda", dev_idx)
    if ws > 1 or ("MASTER_ADDR" in os.environ and "WORLD_SIZE" in os.environ):
        # NCCL when every rank owns a GPU (the normal case, also a 1-rank torchrun launch);
        # gloo only for the control plane when ranks share a device (a functional multi-rank
        # run on a 1-GPU box).
        if ndev >= ws:
            tdist.init_process_group("nccl", device_id=dev)
        else:
            tdist.init_process_group("gloo")
    local = dev_idx

    aliased = args.alias_gb > 0 and wl.table_bytes > args.alias_gb * 1e9
    avail = mem_available()
    if ws == 1 and not aliased and avail and wl.table_bytes > 0.9 * avail:
        log(f"error: the {wl.table_bytes / 1e9:.0f} GB table does not fit the {avail / 1e9:.0f} GB of "
            f"available host RAM; use --alias-gb or a row-scaled workload (name@scale)")
        sys.exit(4)
    if args.host_tier and (aliased or (ws == 1 and avail and 2 * wl.table_bytes > 0.85 * avail)):
        log("host tier off: it needs another full copy of the table in host RAM")
        args.host_tier = False
    table = setup_table(wl, rank, ws, tdist, args.alias_gb)
    unpin_alias = pin_alias_copies(table) if isinstance(table, synth.AliasedHostTable) else None
    t0 = time.time()
    h = synth.hotness(wl)
    log(f"hotness in {time.time() - t0:.1f}s")
    C = wl.capacity_rows
    cfg = make_config(wl.num_rows, wl.row_bytes, C, num_gpus=ws, rank=rank, device=local,
                      policy=args.policy, host_sms=args.host_sms, peer_sms=args.peer_sms)
    t0 = time.time()
    plan, order = solve(cfg, h)
    log(f"solve in {time.time() - t0:.1f}s: k={plan.k} band_end={plan.band_end} z={plan.z:.3e}")
    del h
    t0 = time.time()
    tier = False
    if args.host_tier:
        tier = True  # N = 1: the ctx builds its own rank-ordered host tier
        if ws > 1:   # one tier per node in /dev/shm, filled by rank 0, mapped by all
            from paper_conf_sosp_songz0c23_b200 import fill_host_tier, host_tier_rows
            trows = host_tier_rows(plan, wl.num_rows)
            tpath = f"/dev/shm/ugache_tier_{wl.name}_{os.environ.get('MASTER_PORT', '0')}"
            if rank == 0:
                tier = synth.HostTable(max(trows, 1), wl.row_bytes, shm_path=tpath, create=True)
                fill_host_tier(cfg, order, plan, table, tier)
            tdist.barrier()
            if rank != 0:
                tier = synth.HostTable(max(trows, 1), wl.row_bytes, shm_path=tpath, create=False)
    from paper_conf_sosp_songz0c23_b200._abi import UGACHE_ENOMEM, UGacheError
    try:
        cache = UGache(table, wl.num_rows, wl.row_bytes, C, num_gpus=ws, rank=rank, device=local,
                       policy=args.policy, plan=plan, order=order, host_sms=args.host_sms,
                       peer_sms=args.peer_sms, host_tier=tier)
        ok = 1.0
    except UGacheError as e:
        if e.status != UGACHE_ENOMEM or tier is False:
            raise
        log(f"init with the host tier failed ({e}); every rank retries without it")
        ok = 0.0
    if ugdist.sum_over_ranks(ok) < ws:   # all ranks run the same configuration
        if ok:
            cache.close()
        args.host_tier = False
        tier = False
        cache = UGache(table, wl.num_rows, wl.row_bytes, C, num_gpus=ws, rank=rank, device=local,
                       policy=args.policy, plan=plan, order=order, host_sms=args.host_sms,
                       peer_sms=args.peer_sms, host_tier=False)
    log(f"init (register host table, location table, slab) in {time.time() - t0:.1f}s")
    ugdist.connect(cache, order=order)
    del order
    stream = torch.cuda.Stream(device=dev)
    t0 = time.time()
    cache.fill(stream)
    stream.synchronize()
    ugdist.barrier()
    log(f"fill in {time.time() - t0:.2f}s")
    calibration = None
    if args.calibrate:
        # A0 (ugache_calibrate) on every rank at the same time: the host link and each GPU's
        # NVLink egress carry the load of all G readers.  Reported, not applied:
        # the shipped dedication is the workload calibration.
        ugdist.barrier()
        t0 = time.time()
        cal = cache.calibrate()
        calibration = {k: v for k, v in cal.items()}
        calibration["host_curve_gbs"] = [(k_, b / 1e9) for k_, b in cal["host_curve"]]
        calibration["peer_curve_gbs"] = [(k_, b / 1e9) for k_, b in cal["peer_curve"]]
        del calibration["host_curve"], calibration["peer_curve"]
        log(f"calibration in {time.time() - t0:.2f}s: host_sms {cal['host_sms']} "
            f"({cal['bw_host'] / 1e9:.1f} GB/s), peer_sms {cal['peer_sms']}")
        if ws > 1 and cal["peer_sms"] > 0 and not args.peer_sms:
            # SMs per peer = the tolerance measured under all-to-all
            # load; the SMs left over start on local work (host SMs stay the workload value)
            cache.set_dedication(0, int(ugdist.max_over_ranks(float(cal["peer_sms"]))))
            calibration["applied_peer_sms"] = True
    if args.mode == "random":
        cache.set_mode("random")
    cache.set_stream(args.stream)
    cache.set_inline(host=args.inline != "none", peers=args.inline == "all")

    # Distinct batches, used in order by every loop below (a cursor cycles over them): a
    # batch comes back only after >= --batches other extracts, so no step reuses a recent
    # batch's host rows or their address translations (on this box a host row read again
    # within ~8 batches is served much faster -- DESIGN.md section 7).
    nbat = max(1, args.batches, args.warmup + args.steps)
    batches = make_batches(wl, rank, nbat)
    n = len(batches[0])
    R = wl.row_bytes
    dkeys = [torch.from_numpy(b).to(dev) for b in batches]
    out = torch.empty((n, R), dtype=torch.uint8, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    cursor = [0]

    def next_batch():
        j = cursor[0] % len(dkeys)
        cursor[0] += 1
        return j

    def step(i, timed):
        with torch.cuda.stream(stream):
            flush.fill_(i & 0xFF)  # evict L2 between steps (outside the events)
            # ~50 us of device spin, also outside the events: the host enqueues the step
            # while the GPU is busy, so the events time the step's device work, not the
            # Python/launch latency (that is in the e2e number)
            torch.cuda._sleep(100_000)
        if timed:
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record(stream)
        cache.extract(dkeys[i], out, stream)
        if timed:
            e.record(stream)
            return s, e
        return None

    # ---- warm-up: W steps back to back --------------------------------------------------
    for i in range(args.warmup):
        cache.extract(dkeys[next_batch()], out, stream)
    stream.synchronize()
    ugdist.barrier()
    torch.cuda.synchronize()
    clocks = Clocks(local) if (rank == 0 and not args.no_clocks) else None  # every GPU of the node
    time.sleep(0.3 if clocks else 0)

    # ---- timed region (the line's value): K steps back to back --------------------------
    # Steady state, as an application streams batches: no L2 flush between steps -- every
    # step touches far more than the 126 MB L2 (the batch's rows read and written, its
    # location-table lines), and every step extracts a batch no recent step used -- and
    # no per-step host synchronisation; CUDA events between consecutive steps time each step
    # on the device.  The cold-L2 variant (256 MiB flush before every step) is `cold_l2`.
    cache.enable_timing(False)
    evs, paths = [], []
    launches = 0
    marks = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]
    with torch.cuda.stream(stream):
        # ~1 ms of device spin before the first mark (outside the timed region) lets the
        # host queue the steps ahead of the device, so small batches are not timed at the
        # Python enqueue rate
        torch.cuda._sleep(2_000_000)
    marks[0].record(stream)
    for i in range(args.steps):
        cache.extract(dkeys[next_batch()], out, stream)
        marks[i + 1].record(stream)
        evs.append((marks[i], marks[i + 1]))
        launches += cache.last_launch_count()
        paths.append(cache.last_extract_path())
    stream.synchronize()
    torch.cuda.synchronize()
    ugdist.barrier()
    clk = clocks.stop() if clocks else None
    step_ms = [a.elapsed_time(b) for a, b in evs]
    # a multi-GPU step lasts as long as its slowest rank: per-step max over ranks
    step_max = ugdist.gather_rows(step_ms).max(axis=0)
    max_total_s = ugdist.max_over_ranks(sum(step_ms) / 1e3)
    bytes_all = ugdist.sum_over_ranks(float(args.steps * n * R))
    value = bytes_all / max_total_s / 1e9

    # kernel pass (steady state too: no flush): the library's own events around its launch
    # and the fused kernel's %globaltimer phase split, for the per-kernel roofline
    loc_ms, gat_ms, phases, timeline = [], [], [], None
    cache.enable_timing(True)
    for i in range(args.steps):
        cache.extract(dkeys[next_batch()], out, stream)
        a, b = cache.last_batch_timing()
        loc_ms.append(a)
        gat_ms.append(b)
        if cache.last_extract_path() == "fused":
            phases.append(cache.last_batch_phases())
            timeline = cache.last_batch_timeline()
    stream.synchronize()
    cache.enable_timing(False)
    role_timeline = role_summary(timeline, ws, rank) if phases else None
    log("per-step ms (steady state): " + " ".join(f"{x:.3f}" for x in step_ms))

    # ---- cold L2: the same steps with a 256 MiB flush + ~50 us spin before each -----------
    # (outside the events), per-source counts of every step
    cold_ms, per_src = [], []
    ugdist.barrier()
    for i in range(args.steps):
        ev = step(next_batch(), True)
        per, _ = cache.last_batch_stats()  # syncs this step (after its end event)
        per_src.append(per)
        cold_ms.append(ev[0].elapsed_time(ev[1]))
    cold_max = ugdist.gather_rows(cold_ms).max(axis=0)
    cold_total_s = ugdist.max_over_ranks(sum(cold_ms) / 1e3)
    cold_value = bytes_all / cold_total_s / 1e9
    log("per-step ms (cold L2): " + " ".join(f"{x:.3f}" for x in cold_ms))
    tp_ms = float(np.mean(cold_max))

    # ---- host-only reference: the same kernels on just this batch's host keys ---------
    # (how close the whole step is to the time its host rows alone take on this box; the
    # host source is translation-bound here)
    host_only = None
    if args.extra and args.mode == "factored":
        loc, _ = cache.export_placement()
        hks = []
        for _ in range(args.steps):             # the host keys of the next distinct batches
            b = batches[next_batch()]
            hks.append(np.ascontiguousarray(b[(loc[b] >> np.uint64(56)) == np.uint64(ws)]))
        del loc
        if all(len(h_) for h_ in hks):
            hmax = max(len(h_) for h_ in hks)
            hout = torch.empty((hmax, R), dtype=torch.uint8, device=dev)
            dhks = [torch.from_numpy(h_).to(dev) for h_ in hks]
            hms, hrows = [], 0
            for i, dhk in enumerate(dhks):
                with torch.cuda.stream(stream):
                    flush.fill_(i & 0xFF)
                    torch.cuda._sleep(100_000)
                hs, he = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                hs.record(stream)
                cache.extract(dhk, hout, stream)
                he.record(stream)
                stream.synchronize()
                hms.append(hs.elapsed_time(he))
                hrows += dhk.numel()
            host_only = {"host_keys": hrows / len(dhks), "ms": statistics.mean(hms),
                         "host_gbs": hrows * R / (sum(hms) / 1e3) / 1e9,
                         "path": cache.last_extract_path(),
                         "how": "extracts of only the host keys of distinct batches, same kernels, "
                                "flush and spin as cold_l2"}
            del dhks, hout

    # ---- parity on the full-size batch (every key, byte for byte) -------------------
    # Against the table generator itself (synth: row k's words are a function of k), a
    # property that holds at any size: the oracle stays confined to the cpu_baseline leg.
    def expected_rows(keys):
        k = np.asarray(keys, dtype=np.int64)
        if isinstance(table, synth.AliasedHostTable):
            k = k % table.phys_rows
        return synth.rows_for_keys(k, wl.num_rows, R)

    parity = None
    if not args.no_verify:
        cache.extract(dkeys[0], out, stream)
        stream.synchronize()
        ref = expected_rows(batches[0])
        parity = "bit-exact" if np.array_equal(out.cpu().numpy(), ref) else "MISMATCH"
        del ref

    # ---- e2e through the public API with pinned host buffers -------------------------
    # Default path: the kernels read the pinned keys and write the pinned output in place
    # (zero-copy over PCIe); also timed with staging (H2D copy + extract + D2H copy).
    hkeys = [torch.from_numpy(b).pin_memory() for b in batches]
    hout = torch.empty((n, R), dtype=torch.uint8).pin_memory()
    cache.enable_timing(False)

    def e2e_run(staged):
        cache.set_stage_host_io(staged)
        cache.extract(hkeys[next_batch()], hout, stream)  # warm-up (staging buffers)
        stream.synchronize()
        ms = []
        for i in range(args.e2e_steps):
            with torch.cuda.stream(stream):
                flush.fill_(i & 0xFF)
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record(stream)
            cache.extract(hkeys[next_batch()], hout, stream)
            e.record(stream)
            stream.synchronize()
            ms.append(s.elapsed_time(e))
        cache.set_stage_host_io(False)
        return ms

    e2e_full_ms = e2e_run(False)
    e2e_staged_ms = e2e_run(True)
    e2e_parity = None
    if not args.no_verify:
        cache.extract(hkeys[0], hout, stream)
        stream.synchronize()
        ref = expected_rows(batches[0])
        e2e_parity = "bit-exact" if np.array_equal(hout.numpy(), ref) else "MISMATCH"
        del ref
    # Primary e2e = the embedding-layer call as an application makes it: keys
    # come from pinned host memory, the rows land in HBM where the dense model consumes them,
    # and the host reads back the step's metric (per-source counts + bad keys, which also
    # synchronises).  Host wall clock around the whole call sequence.
    e2e_ms = []
    for i in range(args.e2e_steps + 1):
        with torch.cuda.stream(stream):
            flush.fill_(i & 0xFF)
        stream.synchronize()
        t0 = time.perf_counter()
        cache.extract(hkeys[next_batch()], out, stream)
        per_e2e, bad_e2e = cache.last_batch_stats()
        dt = (time.perf_counter() - t0) * 1e3
        if i:
            e2e_ms.append(dt)
    # Pipelined e2e = the same calls inside an application's input pipeline: step i + 1's keys
    # are copied host -> device (pinned, cudaMemcpyAsync on a copy stream) while step i
    # extracts, as a training loop's data loader prefetches; every step's key copy and its
    # stats readback are inside the timed region (host wall clock over all steps, distinct
    # batches).  The key bytes then share the PCIe link with the host rows instead of
    # delaying the locate pass (the host rows leave ~12 GB/s of the link unused, DESIGN.md
    # section 7).
    kp = max(args.e2e_steps, 10)
    copy_stream = torch.cuda.Stream()
    dkb = [torch.empty(n, dtype=torch.int64, device=dev) for _ in range(2)]
    ev_copy = [torch.cuda.Event() for _ in range(2)]
    order_p = [next_batch() for _ in range(kp)]
    stream.synchronize()
    ugdist.barrier()
    t0 = time.perf_counter()
    with torch.cuda.stream(copy_stream):
        dkb[0].copy_(hkeys[order_p[0]], non_blocking=True)
        ev_copy[0].record(copy_stream)
    for i in range(kp):
        stream.wait_event(ev_copy[i % 2])
        cache.extract(dkb[i % 2], out, stream)
        if i + 1 < kp:   # buffer (i + 1) % 2 was read by step i - 1, whose stats were read back
            with torch.cuda.stream(copy_stream):
                dkb[(i + 1) % 2].copy_(hkeys[order_p[i + 1]], non_blocking=True)
                ev_copy[(i + 1) % 2].record(copy_stream)
        per_p, bad_p = cache.last_batch_stats()    # the step's result; synchronises step i
    e2e_pipe_s = time.perf_counter() - t0
    e2e_pipe_parity = None
    if not args.no_verify:
        ref = expected_rows(batches[order_p[-1]])
        e2e_pipe_parity = "bit-exact" if np.array_equal(out.cpu().numpy(), ref) else "MISMATCH"
        del ref
    e2e_pipe_value = ugdist.sum_over_ranks(float(kp * n * R)) / ugdist.max_over_ranks(e2e_pipe_s) / 1e9
    stats_bytes = (ws + 2) * 8
    e2e_total = ugdist.max_over_ranks(sum(e2e_ms) / 1e3)
    e2e_bytes = ugdist.sum_over_ranks(float(args.e2e_steps * n * R))
    e2e_value = e2e_bytes / e2e_total / 1e9
    e2e_full_value = e2e_bytes / ugdist.max_over_ranks(sum(e2e_full_ms) / 1e3) / 1e9
    e2e_staged_value = e2e_bytes / ugdist.max_over_ranks(sum(e2e_staged_ms) / 1e3) / 1e9

    # ---- optional FEM ablation: random dispatch through the same locate table -------
    ablation = None
    if args.extra and args.mode == "factored":
        cache.set_mode("random")
        cache.enable_timing(False)  # same event placement as the timed factored steps
        for i in range(2):
            cache.extract(dkeys[next_batch()], out, stream)
        rmarks = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]
        with torch.cuda.stream(stream):
            torch.cuda._sleep(2_000_000)
        rmarks[0].record(stream)
        rev = []
        for i in range(args.steps):           # steady state, as the timed steps
            cache.extract(dkeys[next_batch()], out, stream)
            rmarks[i + 1].record(stream)
            rev.append((rmarks[i], rmarks[i + 1]))
        stream.synchronize()
        rms = [a.elapsed_time(b) for a, b in rev]
        rcold = []
        for i in range(args.steps):           # cold L2, as cold_l2
            r = step(next_batch(), True)
            stream.synchronize()
            rcold.append(r[0].elapsed_time(r[1]))
        cache.set_mode("factored")
        ablation = {"random_dispatch_ms_per_step": statistics.mean(rms),
                    "factored_ms_per_step": statistics.mean(step_ms),
                    "cold_l2": {"random_dispatch_ms_per_step": statistics.mean(rcold),
                                "factored_ms_per_step": statistics.mean(cold_ms)}}

    # ---- roofline --------------------------------------------------------------------
    peaks = measured_peaks()
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    hbm_src = "MEASURED_PEAKS.json hbm_gbs" if "hbm_gbs" in peaks else "B200_PROFILING.md fallback"
    # PCIe reference measured on every rank at once (all local GPUs reading host memory
    # concurrently, as during the timed steps): each rank's own pinned-H2D copy rate
    ugdist.barrier()
    pcie = pcie_h2d_peak(torch)
    nvl = NVLINK_GBS
    kb = 8 if dkeys[0].dtype == torch.int64 else 4
    path = statistics.mode(paths)
    # the timed kernel: K2 alone (two launches) or the whole fused / single-pass launch
    kern_ms = [a + b for a, b in zip(loc_ms, gat_ms)] if launches == args.steps else list(gat_ms)
    per = np.mean(np.stack(per_src), axis=0)
    # every rank's numbers, so the batch roofline is the max over GPUs
    mine = np.concatenate([per.astype(np.float64),
                           [n, statistics.mean(kern_ms), statistics.mean(loc_ms), statistics.mean(step_ms),
                            pcie, tp_ms]])
    allr = ugdist.gather_rows(mine)
    P = allr[:, :ws + 1]
    n_all = allr[:, ws + 1]
    kern_all, loc_all, step_all, pcie_all = allr[:, ws + 2], allr[:, ws + 3], allr[:, ws + 4], allr[:, ws + 5]
    rl = batch_roofline(P, n_all, R, kb, path, hbm, pcie_all, nvl)
    slow = int(np.argmax(kern_all))            # the rank whose kernel sets the batch time
    kr = rl["ranks"][slow]
    bound = kr["kernel_bound"]
    kbytes = kr["kernel_bytes"][bound]
    peak = {"hbm": hbm, "pcie": pcie_all[slow], "nvlink_in": nvl, "nvlink_out": nvl}[bound]
    psrc = {"hbm": hbm_src,
            "pcie": "live cudaMemcpy pinned H2D 1 GiB best-of-10 on every rank at once, this run",
            "nvlink_in": "B200_PROFILING.md measured peer copy",
            "nvlink_out": "B200_PROFILING.md measured peer copy"}[bound]
    gat_s = kern_all[slow] / 1e3
    achieved = kbytes / gat_s / 1e9
    unit = "GB/s"
    kname = {"single_pass": "stream_extract_kernel", "fused": "fused_extract_kernel"}.get(
        path, "factored_gather_kernel")
    n_local, n_host = float(per[rank]), float(per[ws])
    n_peer = float(per.sum() - n_local - n_host)
    ms_per_step = float(np.mean(step_max))
    t_roof = rl["t_roof_s"]
    traffic = traffic_pcie = traffic_src = None
    try:  # per-launch DRAM traffic of the kernel from the committed ncu capture of this config
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            recs = json.load(f)[wl.name][kname]
        c_run = args.cache_ratio if args.cache_ratio is not None else wl.cache_ratio
        for rec in (recs if isinstance(recs, list) else [recs]):
            if (abs(rec.get("cache_ratio", wl.cache_ratio) - c_run) < 1e-9 and
                    bool(rec.get("host_tier", False)) == bool(args.host_tier) and rec.get("n_gpus", 1) == ws):
                traffic, traffic_pcie, traffic_src = rec["dram_bytes"], rec.get("pcie_read_bytes"), rec["source"]
                break
    except Exception:
        pass
    # duplicate-aware variant: source reads counted per unique row of the
    # batch (repeats are L2 hits), against the same bandwidths (this rank's batch)
    uniq = len(np.unique(batches[args.warmup % len(batches)]))
    dup_aware = None
    if uniq < n:
        fu = uniq / n
        mr = rl["ranks"][rank]
        u_hbm = n_local * fu * R + n * R + n * (kb + 8) + (16 * n if path != "single_pass" else n_peer * 16)
        u_roof = max(u_hbm / (hbm * 1e9), mr["t_s"]["pcie"] * fu, mr["t_s"]["nvlink_in"] * fu)
        dup_aware = {"unique_keys": uniq, "unique_frac": fu, "t_roof_us": u_roof * 1e6,
                     "frac": u_roof / (ms_per_step / 1e3),
                     "note": "source bytes scaled by the batch's unique fraction (per-source mix assumed "
                             "the same for repeats); output bytes stay n * R"}
    if host_only:
        host_only["step_over_host_only"] = tp_ms / host_only["ms"]   # both cold L2
    line = {
        "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": ws, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": config_dict(args, wl, ws),
        "roofline": {"bound": "pcie" if bound == "pcie" else ("hbm" if bound == "hbm" else "nvlink"),
                     "term": bound, "achieved": achieved, "peak": peak, "unit": unit,
                     "frac": achieved / peak if peak else None, "traffic": traffic,
                     "traffic_pcie_read": traffic_pcie, "traffic_source": traffic_src,
                     "algorithmic_bytes": kr["kernel_bytes"],
                     "kernel": kname + {"fused": " (K1 locate+bucket and K2 gather, one cooperative launch)",
                                        "single_pass": " (K3: locate + copy in one pass, no grid barrier)"}.get(path, ""),
                     "path": path, "rank": slow,
                     "random_row_peak": ({"peak": max(b for _, b in calibration["host_curve_gbs"]),
                                          "frac": achieved / max(b for _, b in calibration["host_curve_gbs"]),
                                          "source": "ugache_calibrate this run: best of the host-source "
                                                    "curve (sorted uniform random rows, k SMs swept)"}
                                         if bound == "pcie" and calibration and calibration["host_curve_gbs"]
                                         else None),
                     "peak_source": psrc,
                     "kernel_ms": kern_all[slow],
                     "how": "algorithmic bytes of the kernel's bounding term on the rank with the longest "
                            "kernel time, / that rank's mean kernel time (CUDA events on the extract stream)"},
        "source_mix_roofline": {"t_roof_us": t_roof * 1e6, "t_step_us": ms_per_step * 1e3,
                                "frac": t_roof / (ms_per_step / 1e3),
                                "bounding_rank": rl["bounding_rank"],
                                "terms_us": {k: v * 1e6 for k, v in rl["ranks"][rl["bounding_rank"]]["t_s"].items()},
                                "bw_gbs": {"hbm": hbm, "pcie": float(np.min(pcie_all)), "nvlink": nvl},
                                "how": "T_roof = max over GPUs g of max(HBM bytes incl. rows served to peers "
                                       "/ BW_HBM, NVLink ingress / BW_NVL, NVLink egress (rows peers read "
                                       "from g) / BW_NVL, host rows / BW_PCIe(g)); t_step = mean over steps "
                                       "of the max over ranks"},
        "per_source_keys": {"local": round(n_local, 2), "peer": round(max(n_peer, 0.0), 2), "host": round(n_host, 2)},
        "per_rank": ({"keys_from_source": P.tolist(), "kernel_ms": kern_all.tolist(),
                      "step_ms": step_all.tolist(), "pcie_peak_gbs": pcie_all.tolist(),
                      "t_roof_us": [r_["t_roof_s"] * 1e6 for r_ in rl["ranks"]]} if ws > 1 else None),
        "ms_p50": float(np.percentile(step_max, 50)), "ms_p99": float(np.percentile(step_max, 99)),
        "cold_l2": {"ms_per_step": tp_ms, "value": cold_value, "unit": "GB/s",
                    "ms_p50": float(np.percentile(cold_max, 50)), "ms_p99": float(np.percentile(cold_max, 99)),
                    "roofline_frac": (kr["kernel_bytes"][bound] / (tp_ms / 1e3) / 1e9) / peak if peak else None,
                    "how": "the same K steps with a 256 MiB L2-flush write and a ~50 us device spin "
                           "before each (outside the events), CUDA events per step, max over ranks; "
                           "roofline_frac = the kernel's bounding-term bytes / the cold step time / peak"},
        "duplicate_aware": dup_aware,
        "host_only": host_only,
        "kernel_ms": {"locate_bucket": float(np.max(loc_all)),
                      "factored_gather": float(np.max(kern_all - (loc_all if launches == args.steps else 0))),
                      "how": "max over ranks of each rank's mean"},
        "fused_phases_ms": ({"locate_done": statistics.mean(p[0] for p in phases),
                             "host_ordered": statistics.mean(p[1] for p in phases),
                             "host_copies_done": statistics.mean(p[2] for p in phases),
                             "last_cta_located": statistics.mean(p[3] for p in phases),
                             "launch_end": statistics.mean(p[4] for p in phases),
                             "how": "%globaltimer stamps inside the fused kernel, ms from its start"}
                            if phases else None),
        "role_timeline_us": role_timeline,
        "e2e": {"value": e2e_pipe_value, "unit": "GB/s", "h2d_bytes_per_step": n * 8,
                "d2h_bytes_per_step": stats_bytes, "ms_per_step": ugdist.max_over_ranks(e2e_pipe_s) / kp * 1e3,
                "steps": kp, "parity": e2e_pipe_parity,
                "path": "input pipeline: pinned host keys -> HBM (cudaMemcpyAsync on a copy stream, "
                        "step i+1's keys during step i) -> UGache.extract (rows in HBM) -> "
                        "ugache_last_batch_stats readback each step; host wall clock over all steps",
                "in_place": {"value": e2e_value, "unit": "GB/s", "ms_per_step": statistics.mean(e2e_ms),
                             "path": "UGache.extract(pinned host keys -> HBM rows) + ugache_last_batch_stats "
                                     "readback per step (host wall clock, L2 flushed and synchronised "
                                     "before each step); the locate kernel reads the pinned keys in place"},
                "full_readback": {"value": e2e_full_value, "unit": "GB/s",
                                  "d2h_bytes_per_step": n * R,
                                  "ms_per_step": statistics.mean(e2e_full_ms),
                                  "path": "pinned host keys and pinned host out: kernels write "
                                          "the rows in place over PCIe (CUDA events)",
                                  "parity": e2e_parity},
                "staged_readback": {"value": e2e_staged_value,
                                    "ms_per_step": statistics.mean(e2e_staged_ms),
                                    "path": "H2D keys + extract + D2H rows (cudaMemcpyAsync)"}},
        "gpu_launches": int(ugdist.sum_over_ranks(float(launches))),
        "clocks": clk,
        "parity": parity,
        "calibration": calibration,
        "plan": {"k": plan.k, "band_end": plan.band_end, "capacity_rows": plan.capacity_rows,
                 "host_sms": plan.host_sms, "peer_sms": plan.peer_sms,
                 "z_model_us": plan.z * 1e6, "z_replication_us": plan.z_replication * 1e6,
                 "z_partition_us": plan.z_partition * 1e6},
    }
    if ablation:
        line["fem_ablation"] = ablation

    # ---- CPU oracle baseline (rank 0, N=1 only, bounded sample, after GPU timing) ----
    if rank == 0 and ws == 1:
        import oracle   # the one place the product bench runs the oracle: cpu_baseline
        out_np = np.empty((n, R), dtype=np.uint8)
        t_end = time.perf_counter() + args.cpu_seconds
        done, cpu_t = 0, 0.0
        while time.perf_counter() < t_end or done == 0:
            b = batches[done % len(batches)]
            t = time.perf_counter()
            oracle.gather(table.ptr, wl.num_rows, R, b, out_np)
            cpu_t += time.perf_counter() - t
            done += 1
        cores = len(os.sched_getaffinity(0))
        line["cpu_baseline"] = {"value": done * n * R / cpu_t / 1e9, "unit": "GB/s",
                                "cores": cores, "kind": "oracle",
                                "sample": f"{done} batches x {n} keys of {wl.name} "
                                          f"(~{args.cpu_seconds:.0f}s, OpenMP {cores} threads)",
                                "ms_per_batch": cpu_t / done * 1e3}
    if rank == 0:
        print(json.dumps(line), flush=True)
    cache.close()
    ugdist.barrier()
    if unpin_alias:
        unpin_alias()
    for buf in (table, tier):
        if isinstance(buf, (synth.HostTable, synth.AliasedHostTable)):
            path = buf.shm_path
            buf.close()
            if ws > 1 and rank == 0 and path and os.path.exists(path):
                os.unlink(path)
    if tdist.is_initialized():
        tdist.destroy_process_group()


if __name__ == "__main__":
    main()

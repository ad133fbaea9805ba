#!/bin/bash
# One-shot GPU-box probe: host RAM, cores, NUMA, PCIe, GPU attributes, pinned-copy bandwidth.
out=gpurun_out/probe
mkdir -p $out
nvidia-smi -q > $out/nvidia-smi-q.txt 2>&1
nvidia-smi topo -m > $out/topo.txt 2>&1
nproc > $out/nproc.txt; free -g > $out/free.txt; df -h /dev/shm > $out/shm.txt
lscpu > $out/lscpu.txt 2>&1; cat /proc/meminfo > $out/meminfo.txt
numactl -H > $out/numa.txt 2>&1
nvidia-smi --query-gpu=pcie.link.gen.current,pcie.link.gen.max,pcie.link.width.current,pcie.link.width.max --format=csv > $out/pcie.txt 2>&1
python - > $out/torch_probe.txt 2>&1 <<'PY'
import torch, time, os
print("affinity", len(os.sched_getaffinity(0)))
p = torch.cuda.get_device_properties(0)
print(p)
print("memgetinfo", torch.cuda.mem_get_info())
# pinned H2D / D2H copy bandwidth
for gb in (1, 4):
    n = gb << 30
    t0 = time.time(); h = torch.empty(n, dtype=torch.uint8, pin_memory=True); print("pin alloc", gb, "GB", time.time()-t0, "s")
    d = torch.empty(n, dtype=torch.uint8, device="cuda")
    for direction in ("h2d", "d2h"):
        best = 1e9
        for _ in range(5):
            s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
            s.record()
            if direction == "h2d": d.copy_(h, non_blocking=True)
            else: h.copy_(d, non_blocking=True)
            e.record(); torch.cuda.synchronize(); best = min(best, s.elapsed_time(e))
        print(direction, gb, "GB", n / best / 1e6, "GB/s")
    del h, d
# host register timing on mmap'd memory
import ctypes, mmap, numpy as np
cudart = ctypes.CDLL("libcudart.so") if False else None
PY

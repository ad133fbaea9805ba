"""Write the host rows of one gnn_pa batch (G = 1, c = 10 %) in host-tier layout for
tools/host_order_probe.cu: tier row = hotness rank - capacity (synth's Zipf rank is the
hotness rank up to float ties), kept in batch order.  Usage: host_order_probe.py out.bin
[workload] [cache_ratio] [batch]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import synth  # noqa: E402

out = sys.argv[1]
wl = synth.get_workload(sys.argv[2] if len(sys.argv) > 2 else "gnn_pa")
c = float(sys.argv[3]) if len(sys.argv) > 3 else 0.1
b = int(sys.argv[4]) if len(sys.argv) > 4 else 0
C = int(wl.num_rows * c)
keys = synth.make_batch(wl, 0, b)
ranks = synth.key_to_rank(keys, wl.num_rows)          # 0-based Zipf rank
host = ranks[ranks >= C] - C
host.astype(np.uint32).tofile(out)
print(f"{len(keys)} keys, {len(host)} host rows, tier rows {wl.num_rows - C}")

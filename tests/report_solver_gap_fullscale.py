#!/usr/bin/env python3
"""Full-scale companion of report_solver_gap.py (not collected): on gnn_pa itself (111M
entries, Zipf(1.2) unique-batch hotness), the block MILP of milp_solver.py (section 6.3
blocks, HiGHS, 120 s limit) against the default hot-replicate / warm-partition sweep of
ugache_solve, G = 2/4/8, c = 10/20 %.  Output: profiles/r2/solver_gap_fullscale.jsonl."""
import sys, time, json
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import synth
from paper_conf_sosp_songz0c23_b200 import make_config, solve
from paper_conf_sosp_songz0c23_b200.milp_solver import make_blocks, solve_blocks
wl = synth.get_workload('gnn_pa')
h = synth.hotness(wl)
N = wl.num_rows
for G in (2, 4, 8):
    for c in (0.1, 0.2):
        C = int(c * N)
        cfg = make_config(N, 512, C, num_gpus=G)
        t0 = time.time()
        plan, order = solve(cfg, h)
        hs = h[order.astype(np.int64)]
        blocks = make_blocks(hs, G)
        T = (plan.T_local, plan.T_peer, plan.T_host); Rr = (plan.R_local, plan.R_peer, plan.R_host)
        t1 = time.time()
        s, a, zb, msg = solve_blocks(hs, blocks, C, G, T, Rr, time_limit=120)
        print(json.dumps({"G": G, "c": c, "blocks": len(blocks), "z_sweep_us": plan.z*1e6, "k": int(plan.k),
                          "z_block_us": zb*1e6, "block_over_sweep": zb/plan.z, "z_rep_us": plan.z_replication*1e6,
                          "z_part_us": plan.z_partition*1e6, "milp_s": time.time()-t1, "msg": msg[:80]}), flush=True)

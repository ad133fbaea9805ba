# NOTE: UGACHE_STREAM_REG_ROWS (K3 register path rows per step) was measured here and then removed
# (no gain, register spills); K3r (stream_extract_reg_kernel) replaced it -- profiles/r2/k3r/.
# Single pass with a sparse host bucket (G = 1): register path 4 vs 8 rows per step, TMA
# slots, and random dispatch, at 20K / 100K / 213K-key batches (gnn_pa@0.25, alpha 1.2).
o=${1:-gpurun_out/regpath}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
for n in 20000 100000; do
  for v in UGACHE_STREAM_REG_ROWS=4 UGACHE_STREAM_REG_ROWS=8 UGACHE_SPARSE_HOST_REGPATH=0; do
    env $v timeout 600 python tools/placement_grid.py --policies ugache --alphas 1.2 --cache-ratios 0.05 0.2 0.5 --gpus 1 --batch-n $n --random --out $o/n${n}_$v.jsonl > /dev/null 2> $o/n${n}_$v.err
  done
done
for v in UGACHE_STREAM_REG_ROWS=4 UGACHE_STREAM_REG_ROWS=8; do
  env $v timeout 300 python bench.py --workload dlr_criteo@0.15 --cache-ratio 0.1 --no-calibrate --cpu-seconds 0.5 > $o/dlr_$v.json 2> $o/dlr_$v.err
done
python - $o <<'PY'
import json, glob, sys
for f in sorted(glob.glob(sys.argv[1] + "/n*.jsonl")):
    for l in open(f):
        r = json.loads(l)
        print(f.split("/")[-1], r["cache_ratio"], "host", round(r["share"]["host"], 4), r["path"], "ms", round(r["measured_ms"], 4),
              "random", round(r.get("random_dispatch_ms", 0), 4), "" if r["bit_exact"] else "MISMATCH")
for f in sorted(glob.glob(sys.argv[1] + "/dlr_*.json")):
    d = json.loads(open(f).read().strip().splitlines()[-1])
    print(f.split("/")[-1], round(d["ms_per_step"], 4), "cold", round(d["cold_l2"]["ms_per_step"], 4), "random", round(d["fem_ablation"]["random_dispatch_ms_per_step"], 4), d["parity"])
PY

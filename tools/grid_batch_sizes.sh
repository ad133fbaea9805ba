# Anomaly hunt: UGache placement at every batch size x cache ratio x G (fake peers), factored
# vs random dispatch on the same contexts and batches (gnn_pa@0.25, alpha 1.2).
o=${1:-gpurun_out/gridb}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
nvidia-smi --query-gpu=name,clocks.sm --format=csv > $o/smi.txt
for n in 2000 20000 100000 500000; do
  timeout 900 python tools/placement_grid.py --policies ugache --alphas 1.2 --cache-ratios 0.05 0.2 0.5 --gpus 1 2 4 8 --batch-n $n --random --out $o/n$n.jsonl > /dev/null 2> $o/n$n.err; echo "n $n rc $?"
done
python - $o <<'PY'
import json, glob, sys
print("n c G k local/peer/host path factored_ms random_ms model_ms ratio_vs_random")
for f in sorted(glob.glob(sys.argv[1] + "/n*.jsonl"), key=lambda x: int(x.split("/n")[-1].split(".")[0])):
    for l in open(f):
        r = json.loads(l)
        sh = r["share"]
        print(f.split("/n")[-1].split(".")[0], r["cache_ratio"], r["G"], r["k"],
              f"{sh['local']:.3f}/{sh['peer']:.3f}/{sh['host']:.3f}", r["path"],
              f"{r['measured_ms']:.4f}", f"{r.get('random_dispatch_ms', 0):.4f}", f"{r['model_z_ms']:.4f}",
              f"{r['measured_ms'] / r.get('random_dispatch_ms', 1):.2f}", "" if r["bit_exact"] else "MISMATCH")
PY

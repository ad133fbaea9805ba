# K3r (lean register single pass for sparse host buckets with every source inline) vs K3's
# register path (UGACHE_REG_KERNEL_CK=0) vs random dispatch: GPU tests, DLR@0.15 c = 2-20 %,
# tiny, and per-call device time at G = 1.
o=${1:-gpurun_out/k3r}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $o/pytest.txt 2>&1; echo "pytest rc $?" >> $o/pytest.txt
for v in 8 16 0; do
  for c in 0.02 0.1 0.2; do
    UGACHE_REG_KERNEL_CK=$v timeout 300 python bench.py --workload dlr_criteo@0.15 --cache-ratio $c --no-calibrate --cpu-seconds 0.5 > $o/dlr_c${c}_ck$v.json 2> $o/dlr_c${c}_ck$v.err
  done
  UGACHE_REG_KERNEL_CK=$v timeout 300 python bench.py --workload tiny --no-calibrate --cpu-seconds 0.5 > $o/tiny_ck$v.json 2> $o/tiny_ck$v.err
done
python tools/summarize_runs.py $o
for f in $o/dlr_*.json $o/tiny_*.json; do python -c "
import json; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f'.split('/')[-1], 'random', round(d['fem_ablation']['random_dispatch_ms_per_step'],4))"; done
tail -2 $o/pytest.txt

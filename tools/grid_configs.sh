# The other BASELINE configs through the three placements on G fake peers (one B200):
# tiny (G = 2, c = 10 %), DLR@0.15 (c = 5/10/20 %, G = 2/4/8), MAG@0.15 (c = 10/20 %, G = 4/8).
o=${1:-gpurun_out/gridc}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
nvidia-smi --query-gpu=name,clocks.sm --format=csv > $o/smi.txt
timeout 300 python tools/placement_grid.py --workload tiny --alphas 1.2 --cache-ratios 0.1 --gpus 2 --out $o/tiny.jsonl --table $o/tiny.md > /dev/null 2> $o/tiny.err; echo "tiny rc $?"
timeout 1500 python tools/placement_grid.py --workload dlr_criteo@0.15 --alphas 1.2 --cache-ratios 0.05 0.1 0.2 --gpus 2 4 8 --out $o/dlr.jsonl --table $o/dlr.md > /dev/null 2> $o/dlr.err; echo "dlr rc $?"
timeout 1500 python tools/placement_grid.py --workload gnn_mag@0.15 --alphas 1.2 --cache-ratios 0.1 0.2 --gpus 4 8 --out $o/mag.jsonl --table $o/mag.md > /dev/null 2> $o/mag.err; echo "mag rc $?"

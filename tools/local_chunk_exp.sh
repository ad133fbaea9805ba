# Adaptive local chunks + PCIe-bound local path choice: role timelines, back-to-back device
# time by batch size (fake peers), the default gnn_pa bench (c = 10 %, 100 %) and DLR@0.15.
o=${1:-gpurun_out/lc}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_extract.py -m gpu -x -q > $o/pytest.txt 2>&1; echo "pytest rc $?" >> $o/pytest.txt
timeout 600 python tools/role_timeline.py --gpus 1 4 8 --out $o/tl_raw.json > $o/tl.jsonl 2> $o/tl.err
timeout 600 python tools/host_overhead.py --gpus 1 2 4 8 --batch-n 2000 20000 100000 500000 > $o/ovh.jsonl 2> $o/ovh.err
timeout 300 python bench.py --no-calibrate --cpu-seconds 0.5 > $o/pa10.json 2> $o/pa10.err
timeout 300 python bench.py --cache-ratio 1.0 --no-calibrate --cpu-seconds 0.5 > $o/pa100.json 2> $o/pa100.err
timeout 300 python bench.py --workload dlr_criteo@0.15 --cache-ratio 0.1 --no-calibrate --cpu-seconds 0.5 > $o/dlr.json 2> $o/dlr.err
python tools/summarize_runs.py $o

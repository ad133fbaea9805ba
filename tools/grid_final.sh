# Placement grid (BASELINE configs[4]) on the final code, plus the targeted GPU tests.
o=${1:-gpurun_out/grid2}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "sparse_host_bucket or fake_peer or preorder" > $o/pytest.txt 2>&1; echo "pytest rc $?" >> $o/pytest.txt
nvidia-smi --query-gpu=name,clocks.sm --format=csv > $o/smi.txt
timeout 2000 python tools/placement_grid.py --out $o/grid.jsonl --table $o/grid.md > $o/out.txt 2> $o/err.txt; echo "grid rc $?"

# Round-end style check on one B200: build, GPU tests, smoke, default bench, reference arm.
set -x
o=${1:-gpurun_out/check}; mkdir -p $o
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $o/smi.txt
nproc > $o/nproc.txt; free -g >> $o/nproc.txt
python __graft_entry__.py > $o/build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $o/pytest_gpu.txt 2>&1; echo "pytest rc $?" >> $o/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $o/smoke.txt 2>&1; echo "smoke rc $?" >> $o/smoke.txt
timeout 900 python bench.py > $o/bench.json 2> $o/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $o/bench_ref.json 2> $o/bench_ref.err
tail -2 $o/pytest_gpu.txt; tail -c 600 $o/bench.json

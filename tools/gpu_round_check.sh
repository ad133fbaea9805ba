set -x
mkdir -p gpurun_out/r1e
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r1e/smi.txt
python __graft_entry__.py > gpurun_out/r1e/build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r1e/pytest_gpu.txt 2>&1; echo "pytest rc $?" >> gpurun_out/r1e/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1e/smoke.txt 2>&1; echo "smoke rc $?" >> gpurun_out/r1e/smoke.txt
timeout 900 python bench.py > gpurun_out/r1e/bench.json 2> gpurun_out/r1e/bench.err
tail -3 gpurun_out/r1e/bench.json

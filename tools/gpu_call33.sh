set -x
o=gpurun_out/r1zm; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
K='single_pass_parity and (1-12-0-host or 4-1-1-none or 8-1-21-all)'
for tool in memcheck racecheck synccheck; do
  timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool $tool --print-limit 20 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "$K" > $o/$tool.txt 2>&1; echo "rc $?" >> $o/$tool.txt
  tail -4 $o/$tool.txt
done

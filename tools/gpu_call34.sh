set -x
o=gpurun_out/r1zn; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
K='single_pass_parity and (1-12-0-host or 4-1-1-none or 8-1-21-all)'
timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool synccheck --num-cuda-barriers 100000 --print-limit 20 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "$K" > $o/synccheck.txt 2>&1; echo "rc $?" >> $o/synccheck.txt
tail -4 $o/synccheck.txt
timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --print-limit 20 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "test_row_sizes and 512-True" > $o/racecheck_k2bulk.txt 2>&1; echo "rc $?" >> $o/racecheck_k2bulk.txt
tail -4 $o/racecheck_k2bulk.txt

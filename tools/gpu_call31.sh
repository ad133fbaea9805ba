set -x
o=gpurun_out/r1zj; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 300 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "single_pass or stream_auto or timing or fused_and_split" > $o/pytest_new.txt 2>&1; echo "rc $?" >> $o/pytest_new.txt
tail -3 $o/pytest_new.txt
grep -q "rc 0" $o/pytest_new.txt || exit 1
timeout 1200 python tools/fake_peer_paths.py --out $o/fake_peer_paths.json > $o/out.txt 2> $o/err.txt; tail -3 $o/err.txt

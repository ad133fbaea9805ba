set -x
o=gpurun_out/r1zp; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 300 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "single_pass_parity" > $o/pytest_new.txt 2>&1; echo "rc $?" >> $o/pytest_new.txt
tail -2 $o/pytest_new.txt
grep -q "rc 0" $o/pytest_new.txt || exit 1
for pw in 16 8 4 2; do
  UGACHE_STREAM_PEER_WARPS=$pw timeout 900 python tools/fake_peer_paths.py --gpus 4 8 --out $o/fpp_pw$pw.json > /dev/null 2> $o/err_pw$pw.txt
  grep "^{" $o/err_pw$pw.txt | python -c "
import sys,json
for l in sys.stdin:
  d=json.loads(l); print('pw=$pw', d['G'], {k:round(v['ms'],3) for k,v in d['variants'].items() if 'single' in k or k=='two_phase'})"
done

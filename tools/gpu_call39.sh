set -x
o=gpurun_out/r1zt; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 300 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "host_range_ordering or pa_shaped or fused_and_split or early_host_walk or warp_granular" > $o/pytest_new.txt 2>&1; echo "rc $?" >> $o/pytest_new.txt
tail -2 $o/pytest_new.txt
grep -q "rc 0" $o/pytest_new.txt || exit 1
for i in 1 2; do
timeout 900 python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 > $o/bench$i.json 2> $o/bench$i.err
python -c "
import json; d=json.loads(open('$o/bench$i.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['fused_phases_ms'], d['host_only']['ms'])"
done

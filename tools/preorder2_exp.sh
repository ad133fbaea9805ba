# CTA-aggregated pre-ordering scatter: parity tests, then gnn_pa c = 10 % / 30 % (fused,
# dense host bucket) with the phase stamps.
o=${1:-gpurun_out/pre2}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $o/pytest.txt 2>&1; echo "pytest rc $?" >> $o/pytest.txt
for r in 1 2; do
  timeout 300 python bench.py --no-calibrate --cpu-seconds 0.5 > $o/pa10_r$r.json 2> $o/pa10_r$r.err
  timeout 300 python bench.py --cache-ratio 0.3 --no-calibrate --cpu-seconds 0.5 > $o/pa30_r$r.json 2> $o/pa30_r$r.err
done
python tools/summarize_runs.py $o
for f in $o/pa*_r*.json; do python -c "
import json; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', d['fused_phases_ms'])"; done

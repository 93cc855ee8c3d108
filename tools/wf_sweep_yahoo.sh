# Deterministic wavefront on the Yahoo-shaped set over (s, c, order, storage): ms/epoch, frac, RMSE
# usage: bash tools/wf_sweep_yahoo.sh "888" "1776 3552 7680" [--cyclic|""] [fp32|fp16]
for s in $1; do for c in $2; do
  r=$(timeout 400 python bench.py --workload yahoo --schedule wavefront --storage ${4:-fp32} --workers $s --wf-cols $c $3 --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --no-deterministic 2>&1 | tail -1 | python -c "import json,sys
try:
    d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],2), round(d['roofline']['frac'],3), round(d['test_rmse'],4))
except Exception as e: print('failed')")
  echo "s=$s c=$c $3 ${4:-fp32} $r"
done; done

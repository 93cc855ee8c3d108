# Deterministic wavefront (fp32, cyclic) over workers s and column blocks c: ms/epoch, frac, RMSE
# usage: bash tools/wf_sweep.sh "592 768" "6144 8192"
for s in ${1:-768}; do for c in ${2:-6144}; do
  r=$(timeout 300 python bench.py --schedule wavefront --storage fp32 --workers $s --wf-cols $c --cyclic --steps 5 --warmup 2 --no-e2e --no-cpu-baseline --no-deterministic 2>&1 | tail -1 | python -c "import json,sys
try:
    d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],2), round(d['roofline']['frac'],3), round(d['test_rmse'],5))
except Exception as e: print('failed')")
  echo "s=$s c=$c $r"
done; done

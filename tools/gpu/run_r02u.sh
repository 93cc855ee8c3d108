B="python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --schedule wavefront --storage fp32 --grid-a 8 --cyclic"
for sc in "96 1000" "96 2000" "111 1500" "111 2200" "64 2000" "128 2000"; do set -- $sc
$B --workers $1 --wf-cols $2 2>&1 | grep "^{" | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('a8 cyclic s=$1 c=$2', round(d['ms_per_step'],2), d['roofline']['workers'])"
done

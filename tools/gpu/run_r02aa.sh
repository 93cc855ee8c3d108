# Hugewiki: lane geometry (8-B lanes = 32 lanes per worker, 16-B default, 32-B lanes)
B="python bench.py --workload hugewiki --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-deterministic"
for lb in 8 32; do for g in "" "--group-cols --batch-f 4096"; do
$B --lane-bytes $lb $g 2>&1 | grep "^{" | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('lb $lb $g', round(d['ms_per_step'],1), round(d['value']/1e9,3), r['workers'], r['lanes_per_worker'], d['clocks']['sm_mhz'])"
done; done

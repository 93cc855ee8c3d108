# regression check of the deterministic wavefront: round-1 final build (tools/r1snap, commit 32bfaa8) vs HEAD
B="--no-e2e --no-cpu-baseline --no-deterministic --schedule wavefront --workers 888 --wf-cols 7680 --cyclic --steps 4 --warmup 3"
for s in fp16 fp32; do
  (cd tools/r1snap && python bench.py $B --storage $s 2>/dev/null | tail -n 1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('r1 $s', round(d['ms_per_step'],3), round(d['roofline']['sgd_ms_per_epoch'],3), d['clocks'])")
  python bench.py $B --storage $s 2>/dev/null | tail -n 1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('head $s', round(d['ms_per_step'],3), round(d['roofline']['sgd_ms_per_epoch'],3), d['clocks'])"
done

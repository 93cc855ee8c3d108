python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "tma_rating" 2>&1 | tail -3
for st in 0 2; do for w in "--workload netflix" "--workload yahoo" "--workload netflix --storage fp32" "--workload netflix --group-cols --batch-f 1024"; do
python bench.py --no-e2e --no-cpu-baseline --no-deterministic --steps 10 --rating-stage $st $w 2>&1 | grep "^{" | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('rs=$st $w', round(d['ms_per_step'],3), d['roofline']['workers'])"
done; done

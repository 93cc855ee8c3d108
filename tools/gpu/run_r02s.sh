python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "exactly_once or ownership or deterministic_one_epoch" > gpurun_out/r02s_tests.log 2>&1
tail -2 gpurun_out/r02s_tests.log
for i in 1 2; do python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --schedule wavefront --storage fp32 --workers 888 --wf-cols 7680 --cyclic 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('det', d['ms_per_step'], d['roofline']['frac'])"; done

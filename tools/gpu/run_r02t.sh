python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -q -p no:cacheprovider -k "wavefront or deterministic or index or ownership or exactly or staged or multirank or out_of_core" > gpurun_out/r02t_tests.log 2>&1
tail -3 gpurun_out/r02t_tests.log
B="python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --schedule wavefront --storage fp32"
$B --grid-a 8 2>&1 | grep "^{" | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('a8 default', d['ms_per_step'], d['roofline']['workers'])"
$B --grid-a 8 --cyclic 2>&1 | grep "^{" | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('a8 cyclic', d['ms_per_step'], d['roofline']['workers'])"
$B --grid-a 8 --cyclic --workers 111 --wf-cols 444 2>&1 | grep "^{" | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('a8 cyclic s111 c444', d['ms_per_step'], d['roofline']['workers'])"
$B --grid-a 8 --cyclic --workers 96 --wf-cols 1000 2>&1 | grep "^{" | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('a8 cyclic s96 c1000', d['ms_per_step'], d['roofline']['workers'])"

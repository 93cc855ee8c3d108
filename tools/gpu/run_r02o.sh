python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "loss or metrics or ownership or visits or exactly" > gpurun_out/r02o_tests.log 2>&1
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r02o_bench.log 2>&1

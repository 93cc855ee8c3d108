python -m pytest tests/test_gpu_multirank.py tests/test_gpu_bench_contract.py -q -p no:cacheprovider > gpurun_out/r02r_tests.log 2>&1
tail -3 gpurun_out/r02r_tests.log

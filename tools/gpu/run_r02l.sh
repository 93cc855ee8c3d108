python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -q -p no:cacheprovider -k "staged or out_of_core or budget or destroy or failed_load or multirank" > gpurun_out/r02l_tests.log 2>&1
tail -30 gpurun_out/r02l_tests.log

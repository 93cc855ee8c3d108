python -m pytest tests/test_gpu_parity.py -q -k "bit_exact_when or low_precision or elementwise" -p no:cacheprovider > gpurun_out/r02b_tests.log 2>&1
python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider --deselect tests/test_gpu_parity.py > gpurun_out/r02b_tests_rest.log 2>&1
tail -3 gpurun_out/r02b_tests.log gpurun_out/r02b_tests_rest.log

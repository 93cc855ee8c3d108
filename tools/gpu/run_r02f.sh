python -m pytest tests/test_gpu_bench_contract.py -q -p no:cacheprovider -x > gpurun_out/r02f_bench_tests.log 2>&1
python bench.py --emulate-ranks 2 --steps 3 --warmup 3 --fraction 0.002 --e2e-steps 1 --cpu-sample 20000 > gpurun_out/r02f_emul2.log 2>&1

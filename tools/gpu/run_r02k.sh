python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "tma_rating" > gpurun_out/r02k_tests.log 2>&1
for st in 0 1; do
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-deterministic --rating-stage $st > gpurun_out/r02k_netflix_rs$st.log 2>&1
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-deterministic --rating-stage $st --workload yahoo > gpurun_out/r02k_yahoo_rs$st.log 2>&1
done

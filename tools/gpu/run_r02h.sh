for st in 0 1; do
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-deterministic --rating-stage $st > gpurun_out/r02h_netflix_rs$st.log 2>&1
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-deterministic --rating-stage $st --workload yahoo > gpurun_out/r02h_yahoo_rs$st.log 2>&1
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-deterministic --rating-stage $st --k 32 > gpurun_out/r02h_netflixk32_rs$st.log 2>&1
done

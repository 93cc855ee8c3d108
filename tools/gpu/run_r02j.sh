python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "tma" > gpurun_out/r02j_tests.log 2>&1
for st in 0 1; do
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-deterministic --rating-stage $st > gpurun_out/r02j_netflix_rs$st.log 2>&1
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-deterministic --rating-stage $st --workload yahoo > gpurun_out/r02j_yahoo_rs$st.log 2>&1
done
B="python bench.py --steps 1 --warmup 2 --no-e2e --no-cpu-baseline --no-deterministic"
ncu --set full --clock-control none -k regex:k_hogwild -s 2 -c 1 -o /tmp/r02_hog_rs1b -f $B --rating-stage 1 > /dev/null 2>&1
ncu -i /tmp/r02_hog_rs1b.ncu-rep --page raw --csv > gpurun_out/r02_hog_rs1b_raw.csv

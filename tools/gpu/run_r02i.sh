B="python bench.py --steps 1 --warmup 2 --no-e2e --no-cpu-baseline --no-deterministic"
for st in 0 1; do
ncu --set full --clock-control none --import-source on -k regex:k_hogwild -s 2 -c 1 -o /tmp/r02_hog_rs$st -f $B --rating-stage $st > gpurun_out/r02i_ncu$st.log 2>&1
ncu -i /tmp/r02_hog_rs$st.ncu-rep --page raw --csv > gpurun_out/r02_hog_rs${st}_raw.csv
ncu -i /tmp/r02_hog_rs$st.ncu-rep --page details --csv > gpurun_out/r02_hog_rs${st}_details.csv
ncu -i /tmp/r02_hog_rs$st.ncu-rep --page source --csv --print-source sass > gpurun_out/r02_hog_rs${st}_sass.csv 2>/dev/null
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r02i_launches.log 2>&1
ls -la gpurun_out/

# q_v loads through L1 (params.q_cache = 0, reading R28) as the default: GPU tests, bench, ncu
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/r02ai_pytest.log 2>&1; tail -3 gpurun_out/r02ai_pytest.log
python bench.py > gpurun_out/r02ai_bench.log 2>&1; grep "^{" gpurun_out/r02ai_bench.log > gpurun_out/r02ai_bench.json
python -c "import json; d=json.load(open('gpurun_out/r02ai_bench.json')); print('bench', round(d['ms_per_step'],3), round(d['value']/1e9,3), d['test_rmse'], d['config']['q_loads'], d['clocks']); [print(k, round(d[k]['ms_per_step'],3), round(d[k]['value']/1e9,3), d[k]['test_rmse']) for k in ('grouped','row_blocks','q_l2_only','deterministic') if d.get(k)]; print('e2e', d['e2e']['value']/1e9)"
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02ai_launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-deterministic > gpurun_out/r02ai_launchlist.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_hogwild -s 4 -c 1 -o gpurun_out/r02ai_nf $B --steps 1 --warmup 3 > gpurun_out/r02ai_ncu1.log 2>&1
ncu -i gpurun_out/r02ai_nf.ncu-rep --page raw --csv > gpurun_out/r02ai_nf_raw.csv 2>&1
ncu --set full --clock-control none -k regex:k_hogwild -s 4 -c 1 -o gpurun_out/r02ai_nfrb $B --grid-cols 1 --steps 1 --warmup 3 > gpurun_out/r02ai_ncu2.log 2>&1
ncu -i gpurun_out/r02ai_nfrb.ncu-rep --page raw --csv > gpurun_out/r02ai_nfrb_raw.csv 2>&1
ncu --set full --clock-control none -k regex:k_hogwild -s 4 -c 1 -o gpurun_out/r02ai_nf32 $B --k 32 --steps 1 --warmup 3 > gpurun_out/r02ai_ncu3.log 2>&1
ncu -i gpurun_out/r02ai_nf32.ncu-rep --page raw --csv > gpurun_out/r02ai_nf32_raw.csv 2>&1
rm -f gpurun_out/*.ncu-rep

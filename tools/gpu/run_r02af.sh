# row-block references: Yahoo plain vs a x 1 auto (RMSE side by side), ncu of Netflix 4 x 1
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic"
run() { n=$1; shift; $B "$@" > gpurun_out/r02af_$n.log 2>&1; grep "^{" gpurun_out/r02af_$n.log > gpurun_out/r02af_$n.json; python -c "import json,sys; d=json.load(open('gpurun_out/r02af_$n.json')); print('$n', round(d['ms_per_step'],2), round(d['value']/1e9,3), round(d['test_rmse'],4), d['config'].get('grid_a'), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 gpurun_out/r02af_$n.log; }
run yh_plain --workload yahoo --steps 10
run yh_auto --workload yahoo --grid-cols 1 --steps 10
run nf_auto --grid-cols 1 --steps 10
run nf32_plain --storage fp32 --steps 10
run nf32_auto --storage fp32 --grid-cols 1 --steps 10
run hw_auto --workload hugewiki --grid-cols 1 --steps 3 --warmup 3
ncu --set full --clock-control none -k regex:k_hogwild -s 12 -c 1 -o gpurun_out/r02af_nf4 python bench.py --grid-cols 1 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-deterministic > gpurun_out/r02af_ncu.log 2>&1
ncu -i gpurun_out/r02af_nf4.ncu-rep --page raw --csv > gpurun_out/r02af_nf4_raw.csv 2>&1
rm -f gpurun_out/r02af_nf4.ncu-rep

# HEAD verification after the grouped-kernel changes + ncu of the best configuration + strata emulation
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02as_smoke.log 2>&1; echo smoke=$? >> gpurun_out/r02as_smoke.log; tail -n 2 gpurun_out/r02as_smoke.log
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/r02as_pytest.log 2>&1; tail -n 3 gpurun_out/r02as_pytest.log
python bench.py > gpurun_out/r02as_bench.log 2>&1; grep "^{" gpurun_out/r02as_bench.log > gpurun_out/r02as_bench.json
python -c "import json; d=json.load(open('gpurun_out/r02as_bench.json')); print('bench', round(d['ms_per_step'],3), round(d['value']/1e9,3), d['test_rmse'], round(d['roofline']['frac'],3), d['clocks']); [print(k, round(d[k]['ms_per_step'],3), round(d[k]['value']/1e9,3), d[k]['test_rmse']) for k in ('grouped','row_blocks','row_blocks_grouped','q_l2_only','deterministic') if d.get(k)]; print('e2e', d['e2e']['value']/1e9)"
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic"
ncu --set full --clock-control none --import-source on -k regex:k_hogwild -s 3 -c 1 -o gpurun_out/r02as_best $B --grid-cols 1 --group-cols --batch-f 1024 --steps 1 --warmup 3 > gpurun_out/r02as_ncu.log 2>&1
ncu -i gpurun_out/r02as_best.ncu-rep --page raw --csv > gpurun_out/r02as_best_raw.csv 2>&1
ncu -i gpurun_out/r02as_best.ncu-rep --page source --csv > gpurun_out/r02as_best_src.csv 2>&1
rm -f gpurun_out/*.ncu-rep
for G in 4 8; do
  python tools/scale_emulation.py --workload hugewiki --gs $G --no-base --group-cols --batch-f 1024 --out gpurun_out/r02as_scale_hw_grp1024_G$G.json > gpurun_out/r02as_scale_G$G.log 2>&1; tail -n 1 gpurun_out/r02as_scale_G$G.log
done

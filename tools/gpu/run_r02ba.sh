# wavefront register cap 168 as the default: GPU tests, smoke, bench line, deterministic k/precision sweep
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02ba_smoke.log 2>&1; echo smoke=$? >> gpurun_out/r02ba_smoke.log; tail -n 2 gpurun_out/r02ba_smoke.log
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/r02ba_pytest.log 2>&1; tail -n 3 gpurun_out/r02ba_pytest.log
python bench.py > gpurun_out/r02ba_bench.log 2>&1; grep "^{" gpurun_out/r02ba_bench.log > gpurun_out/r02ba_bench.json
python -c "import json; d=json.load(open('gpurun_out/r02ba_bench.json')); print('bench', round(d['ms_per_step'],3), round(d['value']/1e9,3), d['test_rmse'], round(d['roofline']['frac'],3), d['clocks']); [print(k, round(d[k]['ms_per_step'],3), round(d[k]['value']/1e9,3), d[k]['test_rmse'], d[k].get('roofline',{}).get('frac')) for k in ('grouped','row_blocks','row_blocks_grouped','q_l2_only','deterministic') if d.get(k)]; print('e2e', d['e2e']['value']/1e9)"
python tools/sweep.py --name r02ba_det --set det --steps 4 --warmup 3 > gpurun_out/r02ba_det.log 2>&1; cat gpurun_out/r02ba_det.md

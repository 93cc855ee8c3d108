# HEAD verification: smoke, full GPU suite, default bench line, Hugewiki one-GPU line (configs[3] at N = 1)
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02al_smoke.log 2>&1; echo smoke=$? >> gpurun_out/r02al_smoke.log; tail -n 2 gpurun_out/r02al_smoke.log
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/r02al_pytest.log 2>&1; tail -n 3 gpurun_out/r02al_pytest.log
python bench.py > gpurun_out/r02al_bench.log 2>&1; grep "^{" gpurun_out/r02al_bench.log > gpurun_out/r02al_bench.json
python -c "import json; d=json.load(open('gpurun_out/r02al_bench.json')); print('bench', round(d['ms_per_step'],3), round(d['value']/1e9,3), d['test_rmse'], d['roofline']['frac'], d['roofline'].get('dram'), d['clocks']); [print(k, round(d[k]['ms_per_step'],3), round(d[k]['value']/1e9,3), d[k]['test_rmse']) for k in ('grouped','row_blocks','q_l2_only','deterministic') if d.get(k)]; print('e2e', d['e2e']['value']/1e9)"
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r02al_ref.log 2>&1; grep "^{" gpurun_out/r02al_ref.log > gpurun_out/r02al_ref.json; head -c 300 gpurun_out/r02al_ref.json; echo
python bench.py --workload hugewiki --steps 3 --warmup 3 > gpurun_out/r02al_hw.log 2>&1; grep "^{" gpurun_out/r02al_hw.log > gpurun_out/r02al_hw.json
python -c "import json; d=json.load(open('gpurun_out/r02al_hw.json')); print('hw', round(d['ms_per_step'],3), round(d['value']/1e9,3), d['test_rmse'], d['config']['grid_a'], d['clocks'])"

# final round-2 verification at HEAD: smoke, full GPU suite, default bench line, reference arm, launch list
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02aw_smoke.log 2>&1; echo smoke=$? >> gpurun_out/r02aw_smoke.log; tail -n 2 gpurun_out/r02aw_smoke.log
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/r02aw_pytest.log 2>&1; tail -n 3 gpurun_out/r02aw_pytest.log
python bench.py > gpurun_out/r02aw_bench.log 2>&1; grep "^{" gpurun_out/r02aw_bench.log > gpurun_out/r02aw_bench.json
python -c "import json; d=json.load(open('gpurun_out/r02aw_bench.json')); print('bench', round(d['ms_per_step'],3), round(d['value']/1e9,3), d['test_rmse'], round(d['roofline']['frac'],3), d['clocks']); [print(k, round(d[k]['ms_per_step'],3), round(d[k]['value']/1e9,3), d[k]['test_rmse']) for k in ('grouped','row_blocks','row_blocks_grouped','q_l2_only','deterministic') if d.get(k)]; print('e2e', d['e2e']['value']/1e9)"
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r02aw_ref.log 2>&1; grep "^{" gpurun_out/r02aw_ref.log > gpurun_out/r02aw_ref.json; head -c 200 gpurun_out/r02aw_ref.json; echo
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02aw_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/r02aw_launchlist.log 2>&1; echo ncu=$?

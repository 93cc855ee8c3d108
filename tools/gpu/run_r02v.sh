python -m pytest tests -m gpu -q --timeout 2400 -p no:cacheprovider > gpurun_out/r02v_gputests.log 2>&1
tail -3 gpurun_out/r02v_gputests.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
python bench.py > gpurun_out/r02v_bench.log 2>&1
grep "^{" gpurun_out/r02v_bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value']/1e9, d['ms_per_step'], d['roofline']['frac'], d['deterministic']['ms_per_step'], d['grouped']['ms_per_step'], d['e2e']['value']/1e9, d['cpu_baseline']['value'], d['clocks'])"
python bench.py --impl reference --steps 2 --warmup 3 2>&1 | tail -1 | cut -c1-300

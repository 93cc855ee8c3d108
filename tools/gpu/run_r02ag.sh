# a x 1 row blocks in ONE launch per epoch (concatenated chunk list): tests + block-count sweep
python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "row_block or index_structures" > gpurun_out/r02ag_tests.log 2>&1; tail -2 gpurun_out/r02ag_tests.log
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic"
run() { n=$1; shift; $B "$@" > gpurun_out/r02ag_$n.log 2>&1; grep "^{" gpurun_out/r02ag_$n.log > gpurun_out/r02ag_$n.json; python -c "import json,sys; d=json.load(open('gpurun_out/r02ag_$n.json')); print('$n', round(d['ms_per_step'],2), round(d['value']/1e9,3), round(d['test_rmse'],4), d['config'].get('grid_a'), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 gpurun_out/r02ag_$n.log; }
for a in 2 4 8 16 32 64; do run nf_a${a} --grid-a $a --grid-cols 1 --steps 10; done
run nf32_a8 --storage fp32 --grid-a 8 --grid-cols 1 --steps 10
run nf32_a16 --storage fp32 --grid-a 16 --grid-cols 1 --steps 10
for a in 8 16 32; do run yh_a$a --workload yahoo --grid-a $a --grid-cols 1 --steps 10; done
for a in 64 256; do run hw_a$a --workload hugewiki --grid-a $a --grid-cols 1 --steps 3 --warmup 3; done

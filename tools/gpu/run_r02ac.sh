# a x 1 row blocks (R27): Netflix a = 8 resident / ratings staged / ratings + P staged, and the
# paper's Hugewiki 64 x 1 configuration resident and with P out of core
free -g | head -2
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic"
run() { n=$1; shift; $B "$@" > gpurun_out/r02ac_$n.log 2>&1; grep "^{" gpurun_out/r02ac_$n.log > gpurun_out/r02ac_$n.json; python -c "import json,sys; d=json.load(open('gpurun_out/r02ac_$n.json')); print('$n', round(d['ms_per_step'],2), round(d['value']/1e9,3), round(d['test_rmse'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 gpurun_out/r02ac_$n.log; }
run nf_a8x1_s0 --grid-a 8 --grid-cols 1 --steps 10
run nf_a8x1_s1 --grid-a 8 --grid-cols 1 --staged 1 --steps 10
run nf_a8x1_s2 --grid-a 8 --grid-cols 1 --staged 2 --steps 10
run nf_a8_s2 --grid-a 8 --staged 2 --steps 10
run hw_64x1_s0 --workload hugewiki --grid-a 64 --grid-cols 1 --steps 3 --warmup 3
run hw_64x1_s2 --workload hugewiki --grid-a 64 --grid-cols 1 --staged 2 --steps 2 --warmup 1

# a x 1 row blocks (R27): block-count sweep (P-row locality in L2 vs per-launch tails)
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic"
run() { n=$1; shift; $B "$@" > gpurun_out/r02ad_$n.log 2>&1; grep "^{" gpurun_out/r02ad_$n.log > gpurun_out/r02ad_$n.json; python -c "import json,sys; d=json.load(open('gpurun_out/r02ad_$n.json')); print('$n', round(d['ms_per_step'],2), round(d['value']/1e9,3), round(d['test_rmse'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 gpurun_out/r02ad_$n.log; }
for a in 2 4 16 32; do run nf_a${a}x1 --grid-a $a --grid-cols 1 --steps 10; done
run nf_a8x1_grp --grid-a 8 --grid-cols 1 --group-cols --batch-f 1024 --steps 10
run nf_a4x1_grp --grid-a 4 --grid-cols 1 --group-cols --batch-f 1024 --steps 10
run yh_a8x1 --workload yahoo --grid-a 8 --grid-cols 1 --steps 10
run yh_a16x1 --workload yahoo --grid-a 16 --grid-cols 1 --steps 10
for a in 128 256; do run hw_${a}x1 --workload hugewiki --grid-a $a --grid-cols 1 --steps 3 --warmup 3; done
run hw_128x1_grp --workload hugewiki --grid-a 128 --grid-cols 1 --group-cols --batch-f 4096 --steps 3 --warmup 3
run hw_64x1_grp --workload hugewiki --grid-a 64 --grid-cols 1 --group-cols --batch-f 4096 --steps 3 --warmup 3

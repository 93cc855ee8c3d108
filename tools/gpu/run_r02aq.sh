# grouped batches with the batch-unrolled loop (GRP only) + L1 q_v: parity and f / grid sweep
timeout 600 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "grouped or q_loads or one_worker" > gpurun_out/r02aq_tests.log 2>&1; tail -n 2 gpurun_out/r02aq_tests.log
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic --steps 10"
run() { n=$1; shift; $B "$@" > gpurun_out/r02aq_$n.log 2>&1; grep "^{" gpurun_out/r02aq_$n.log > gpurun_out/r02aq_$n.json; python -c "import json,sys; d=json.load(open('gpurun_out/r02aq_$n.json')); print('$n', round(d['ms_per_step'],3), round(d['value']/1e9,3), round(d['test_rmse'],5), d['config'].get('grid_a'), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -n 3 gpurun_out/r02aq_$n.log; }
run nf_plain
for f in 512 1024 2048 4096; do run nf_grp$f --group-cols --batch-f $f; done
run nfrb_grp1024 --group-cols --batch-f 1024 --grid-cols 1
run nfrb2_grp1024 --group-cols --batch-f 1024 --grid-cols 1 --grid-a 2
run nf32_grp1024 --k 32 --group-cols --batch-f 1024
run nf32s_grp1024 --storage fp32 --group-cols --batch-f 1024
run yh_grp1024 --workload yahoo --group-cols --batch-f 1024
run hw11_grp8192 --workload hugewiki --grid-a 1 --group-cols --batch-f 8192 --steps 3 --warmup 3
run hw256_grp1024 --workload hugewiki --grid-cols 1 --grid-a 256 --group-cols --batch-f 1024 --steps 3 --warmup 3
run hw64_grp1024 --workload hugewiki --grid-cols 1 --grid-a 64 --group-cols --batch-f 1024 --steps 3 --warmup 3

# Hugewiki one GPU: column-grouped batch size sweep (hot-column L2 read-modify-write bound)
B="python bench.py --workload hugewiki --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-deterministic"
run() { n=$1; shift; $B "$@" > gpurun_out/r02y_$n.log 2>&1; grep "^{" gpurun_out/r02y_$n.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$n', round(d['ms_per_step'],1), round(d['value']/1e9,3), round(d['test_rmse'],4), r['workers'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 gpurun_out/r02y_$n.log; }
run grp1024 --group-cols --batch-f 1024
run grp2048 --group-cols --batch-f 2048
run grp4096 --group-cols --batch-f 4096
run grp8192 --group-cols --batch-f 8192
run grp4096_rs1 --group-cols --batch-f 4096 --rating-stage 1
run plain1024 --batch-f 1024

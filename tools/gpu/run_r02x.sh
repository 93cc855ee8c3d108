# Hugewiki one-GPU memory-level-parallelism sweep (is the plain kernel latency-bound on P-row misses?)
B="python bench.py --workload hugewiki --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-deterministic"
run() { n=$1; shift; $B "$@" > gpurun_out/r02x_$n.log 2>&1; grep "^{" gpurun_out/r02x_$n.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$n', round(d['ms_per_step'],1), round(d['value']/1e9,3), r['workers'], r['grid'], d['clocks'])"; }
run plain
run pf2 --prefetch 2
run rs1 --rating-stage 1
run rs2 --rating-stage 2
run grp --group-cols --batch-f 1024
run grp_rs2 --group-cols --batch-f 1024 --rating-stage 2
run w2x --workers 23680
ncu --set full --clock-control none -k regex:k_hogwild -s 3 -c 1 -o gpurun_out/r02x_hw $B --steps 1 --warmup 3 > gpurun_out/r02x_ncu.log 2>&1
ncu -i gpurun_out/r02x_hw.ncu-rep --page raw --csv > gpurun_out/r02x_hw_raw.csv 2>&1
rm -f gpurun_out/r02x_hw.ncu-rep

# ncu of the L1 q_v kernel (r02ai skipped past the last launch) + Hugewiki / Yahoo / k = 32 with L1
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic"
run() { n=$1; shift; $B "$@" > gpurun_out/r02aj_$n.log 2>&1; grep "^{" gpurun_out/r02aj_$n.log > gpurun_out/r02aj_$n.json; python -c "import json,sys; d=json.load(open('gpurun_out/r02aj_$n.json')); print('$n', round(d['ms_per_step'],2), round(d['value']/1e9,3), round(d['test_rmse'],5), d['config'].get('grid_a'), d['config'].get('q_loads'), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 gpurun_out/r02aj_$n.log; }
for x in "nf:" "nfrb:--grid-cols 1" "nf32:--k 32"; do n=${x%%:*}; a=${x#*:}
  ncu --set full --clock-control none --import-source on -k regex:k_hogwild -s 3 -c 1 -o gpurun_out/r02aj_$n $B $a --steps 1 --warmup 3 > gpurun_out/r02aj_ncu_$n.log 2>&1
  ncu -i gpurun_out/r02aj_$n.ncu-rep --page raw --csv > gpurun_out/r02aj_${n}_raw.csv 2>&1
  ncu -i gpurun_out/r02aj_$n.ncu-rep --page source --csv > gpurun_out/r02aj_${n}_src.csv 2>&1
done
rm -f gpurun_out/*.ncu-rep
run nf32rb --k 32 --grid-cols 1 --steps 10
run nf32rb_l2 --k 32 --grid-cols 1 --steps 10 --q-cache 1
run yhrb --workload yahoo --grid-cols 1 --steps 10
run nf32s --storage fp32 --steps 10
run nf32s_l2 --storage fp32 --steps 10 --q-cache 1
run hw64 --workload hugewiki --steps 3 --warmup 3
run hw64_l2 --workload hugewiki --steps 3 --warmup 3 --q-cache 1
run hwauto --workload hugewiki --grid-cols 1 --grid-a 256 --steps 3 --warmup 3
run hw11 --workload hugewiki --grid-a 1 --steps 3 --warmup 3

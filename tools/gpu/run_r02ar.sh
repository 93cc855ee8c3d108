# probe: 4 blocks/SM (64 regs) with the unrolled loop for grouped (minb4) and also plain (up_minb4) vs default
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic --steps 10"
run() { n=$1; shift; $B "$@" > gpurun_out/r02ar_$n.log 2>&1; grep "^{" gpurun_out/r02ar_$n.log > gpurun_out/r02ar_$n.json; python -c "import json,sys; d=json.load(open('gpurun_out/r02ar_$n.json')); print('$n', round(d['ms_per_step'],3), round(d['value']/1e9,3), round(d['test_rmse'],5), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -n 3 gpurun_out/r02ar_$n.log; }
for v in base minb4 up_minb4; do
  if [ $v = base ]; then unset MF_LIB; else export MF_LIB=tools/bin/$v.so; fi
  run ${v}_nf; run ${v}_nfgrp --group-cols --batch-f 1024; run ${v}_nfrbgrp --grid-cols 1 --group-cols --batch-f 1024; run ${v}_nfrb --grid-cols 1; run ${v}_yh --workload yahoo; run ${v}_nf32 --k 32; run ${v}_nf32grp --k 32 --group-cols --batch-f 1024
done

# Hogwild row-access cache policy probe (MF_HW_LC; tools/bin/lc*.so): L2-only (.cg, base) vs L1-cached
# q_v / p_u loads (.ca) and write-back stores; ms/epoch and the 15-epoch test RMSE per workload.
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic --steps 10"
for v in base lc1 lc5 lc3 lc15; do
  if [ $v = base ]; then unset MF_LIB; else export MF_LIB=tools/bin/$v.so; fi
  for w in "nf:--workload netflix" "nfrb:--workload netflix --grid-cols 1" "yh:--workload yahoo" "nf32:--workload netflix --k 32"; do
    n=${w%%:*}; a=${w#*:}
    $B $a > gpurun_out/r02ah_${v}_$n.log 2>&1
    grep "^{" gpurun_out/r02ah_${v}_$n.log > gpurun_out/r02ah_${v}_$n.json
    python -c "import json; d=json.load(open('gpurun_out/r02ah_${v}_$n.json')); print('$v $n', round(d['ms_per_step'],3), round(d['value']/1e9,3), round(d['test_rmse'],5), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 gpurun_out/r02ah_${v}_$n.log
  done
done

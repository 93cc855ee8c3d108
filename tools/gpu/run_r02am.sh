# probe: 16-lane group sum through REDUX (split fixed point, per half-warp mask) vs the shfl butterfly
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic --steps 10"
run() { n=$1; shift; $B "$@" > gpurun_out/r02am_$n.log 2>&1; grep "^{" gpurun_out/r02am_$n.log > gpurun_out/r02am_$n.json; python -c "import json,sys; d=json.load(open('gpurun_out/r02am_$n.json')); print('$n', round(d['ms_per_step'],3), round(d['value']/1e9,3), round(d['test_rmse'],5), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -n 3 gpurun_out/r02am_$n.log; }
for v in base redux16; do
  if [ $v = base ]; then unset MF_LIB; else export MF_LIB=tools/bin/$v.so; fi
  run ${v}_nf; run ${v}_nfrb --grid-cols 1; run ${v}_nf32s --storage fp32
done
export MF_LIB=tools/bin/redux16.so
timeout 600 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "one_worker or q_loads or hogwild" > gpurun_out/r02am_tests.log 2>&1; tail -n 5 gpurun_out/r02am_tests.log

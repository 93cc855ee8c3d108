# A/B: batch-unrolled Hogwild sample loop (MF_BATCH_UNROLL=1, product build) vs the rolled loop (0)
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic --steps 10"
run() { n=$1; shift; $B "$@" > gpurun_out/r02ap_$n.log 2>&1; grep "^{" gpurun_out/r02ap_$n.log > gpurun_out/r02ap_$n.json; python -c "import json,sys; d=json.load(open('gpurun_out/r02ap_$n.json')); print('$n', round(d['ms_per_step'],3), round(d['value']/1e9,3), round(d['test_rmse'],5), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -n 3 gpurun_out/r02ap_$n.log; }
for v in unroll1 unroll0; do
  if [ $v = unroll1 ]; then unset MF_LIB; else export MF_LIB=tools/bin/$v.so; fi
  run ${v}_nf; run ${v}_nfrb --grid-cols 1; run ${v}_nf32 --k 32; run ${v}_yh --workload yahoo; run ${v}_nf32s --storage fp32; run ${v}_nf64 --k 64; run ${v}_grp --group-cols --batch-f 1024
done
unset MF_LIB
timeout 600 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "one_worker or q_loads or hogwild or grouped or row_block" > gpurun_out/r02ap_tests.log 2>&1; tail -n 3 gpurun_out/r02ap_tests.log

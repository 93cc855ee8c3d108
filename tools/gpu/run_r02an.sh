# probe: prefetch depth 2 with 3 / 4 resident blocks per SM (MF_HOG_MINB_D2) vs depth 1 at 5
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic --steps 10"
run() { n=$1; shift; $B "$@" > gpurun_out/r02an_$n.log 2>&1; grep "^{" gpurun_out/r02an_$n.log > gpurun_out/r02an_$n.json; python -c "import json,sys; d=json.load(open('gpurun_out/r02an_$n.json')); print('$n', round(d['ms_per_step'],3), round(d['value']/1e9,3), round(d['test_rmse'],5), d['roofline']['workers'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -n 3 gpurun_out/r02an_$n.log; }
run base_nf; run base_nfrb --grid-cols 1; run base_nf32 --k 32
for v in d2minb3 d2minb4; do export MF_LIB=tools/bin/$v.so
  run ${v}_nf --prefetch 2; run ${v}_nfrb --grid-cols 1 --prefetch 2; run ${v}_nf32 --k 32 --prefetch 2; run ${v}_yh --workload yahoo --prefetch 2
done

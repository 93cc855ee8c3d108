# L1 q_v loads: narrow lanes / prefetch 2 / occupancy probes; DSGD strata emulation with L1 (Hugewiki full size)
timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "q_loads or one_worker_elementwise" > gpurun_out/r02ak_tests.log 2>&1; tail -n 2 gpurun_out/r02ak_tests.log
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic --steps 10"
run() { n=$1; shift; $B "$@" > gpurun_out/r02ak_$n.log 2>&1; grep "^{" gpurun_out/r02ak_$n.log > gpurun_out/r02ak_$n.json; python -c "import json,sys; d=json.load(open('gpurun_out/r02ak_$n.json')); print('$n', round(d['ms_per_step'],3), round(d['value']/1e9,3), round(d['test_rmse'],5), d['roofline']['lanes_per_worker'], d['roofline']['workers'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -n 3 gpurun_out/r02ak_$n.log; }
run nf
run nf_p2 --prefetch 2
run nf32
run nf32_lb8 --k 32 --lane-bytes 8
run nf32_p2 --k 32 --prefetch 2
run nf32_lb8p2 --k 32 --lane-bytes 8 --prefetch 2
run nfrb_p2 --grid-cols 1 --prefetch 2
for v in minb6 minb4; do export MF_LIB=tools/bin/$v.so; run nf_$v; run nf32_$v --k 32; run nfrb_$v --grid-cols 1; done; unset MF_LIB
for G in 1 2 4 8; do
  python tools/scale_emulation.py --workload hugewiki --gs $G --no-base --out gpurun_out/r02ak_scale_hw_plain256_G$G.json > gpurun_out/r02ak_scale_plain_G$G.log 2>&1; tail -n 1 gpurun_out/r02ak_scale_plain_G$G.log
  python tools/scale_emulation.py --workload hugewiki --gs $G --no-base --group-cols --batch-f 1024 --out gpurun_out/r02ak_scale_hw_grp1024_G$G.json > gpurun_out/r02ak_scale_grp_G$G.log 2>&1; tail -n 1 gpurun_out/r02ak_scale_grp_G$G.log
done
python tools/scale_emulation.py --workload netflix --gs 1,2,4,8 --out gpurun_out/r02ak_scale_nf_plain.json > gpurun_out/r02ak_scale_nf.log 2>&1; cat gpurun_out/r02ak_scale_nf.log | grep "^{"

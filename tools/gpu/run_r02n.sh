python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "grouped" > gpurun_out/r02n_tests.log 2>&1
B="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-deterministic"
$B > gpurun_out/r02n_base.log 2>&1
for f in 256 512 1024 2048 4096; do $B --group-cols --batch-f $f > gpurun_out/r02n_g$f.log 2>&1; done
$B --workload yahoo > gpurun_out/r02n_ybase.log 2>&1
$B --workload yahoo --group-cols --batch-f 512 > gpurun_out/r02n_yg512.log 2>&1
$B --k 32 > gpurun_out/r02n_k32base.log 2>&1
$B --k 32 --group-cols --batch-f 256 > gpurun_out/r02n_k32g256.log 2>&1
$B --storage fp32 > gpurun_out/r02n_f32base.log 2>&1
$B --storage fp32 --group-cols --batch-f 1024 > gpurun_out/r02n_f32g1024.log 2>&1

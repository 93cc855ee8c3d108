python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "grouped or one_worker or deterministic_one_epoch or staged or adagrad" > gpurun_out/r02m_tests.log 2>&1
B="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-deterministic"
$B > gpurun_out/r02m_base.log 2>&1
for f in 256 512 1024 2048; do $B --group-cols --batch-f $f > gpurun_out/r02m_g$f.log 2>&1; done
$B --batch-f 1024 > gpurun_out/r02m_p1024.log 2>&1
$B --workload yahoo > gpurun_out/r02m_ybase.log 2>&1
$B --workload yahoo --group-cols --batch-f 1024 > gpurun_out/r02m_yg1024.log 2>&1
$B --k 32 > gpurun_out/r02m_k32base.log 2>&1
$B --k 32 --group-cols --batch-f 1024 > gpurun_out/r02m_k32g1024.log 2>&1

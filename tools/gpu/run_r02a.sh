set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -m pytest tests -m gpu -q -x --timeout 1500 -p no:cacheprovider > gpurun_out/r02a_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r02a_tests.log
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r02a_bench_lit.log 2>&1
MF_LIB=tools/bin/fastupd.so python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r02a_bench_fast.log 2>&1
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --schedule wavefront --storage fp16 --workers 888 --wf-cols 7680 --cyclic > gpurun_out/r02a_wf16_lit.log 2>&1
MF_LIB=tools/bin/fastupd.so python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --schedule wavefront --storage fp16 --workers 888 --wf-cols 7680 --cyclic > gpurun_out/r02a_wf16_fast.log 2>&1
tail -3 gpurun_out/r02a_tests.log

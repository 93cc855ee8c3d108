python tools/parity_fraction_probe.py > gpurun_out/r02d_probe.log 2>&1
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r02d_bench.log 2>&1
python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --schedule wavefront --storage fp16 --workers 888 --wf-cols 7680 --cyclic > gpurun_out/r02d_wf16.log 2>&1

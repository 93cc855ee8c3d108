# configs[4] at HEAD: k = 32..256 x fp32/fp16/bf16 on the Netflix shape, plain Hogwild (headline kernel),
# the best Hogwild configuration (4 x 1 rows + grouped f = 1024) and the deterministic wavefront
python tools/sweep.py --name r02at_kprec --set kprec --steps 8 --warmup 3 > gpurun_out/r02at_kprec.log 2>&1
python tools/sweep.py --name r02at_kprec_best --set kprec_best --steps 8 --warmup 3 > gpurun_out/r02at_best.log 2>&1
python tools/sweep.py --name r02at_det --set det --steps 4 --warmup 3 > gpurun_out/r02at_det.log 2>&1
cat gpurun_out/r02at_kprec.md gpurun_out/r02at_kprec_best.md gpurun_out/r02at_det.md

# ncu --set full of the deterministic wavefront, fp16 vs fp32 (k = 128, s = 888, c = 7680, cyclic)
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic --schedule wavefront --workers 888 --wf-cols 7680 --cyclic --steps 1 --warmup 2"
for s in fp16 fp32; do
  ncu --set full --clock-control none --import-source on -k regex:k_wavefront2 -s 2 -c 1 -o gpurun_out/r02ay_$s $B --storage $s > gpurun_out/r02ay_ncu_$s.log 2>&1
  ncu -i gpurun_out/r02ay_$s.ncu-rep --page raw --csv > gpurun_out/r02ay_${s}_raw.csv 2>&1
  ncu -i gpurun_out/r02ay_$s.ncu-rep --page source --csv > gpurun_out/r02ay_${s}_src.csv 2>&1
done
rm -f gpurun_out/*.ncu-rep

python tools/scale_emulation.py --workload hugewiki --fraction 0.5 --epochs 3 --out gpurun_out/scale_hugewiki_half_plain.json > gpurun_out/r02q_plain.log 2>&1
python tools/scale_emulation.py --workload hugewiki --fraction 0.5 --epochs 3 --no-base --group-cols --batch-f 1024 --out gpurun_out/scale_hugewiki_half_grouped1024.json > gpurun_out/r02q_g1024.log 2>&1
python tools/scale_emulation.py --workload hugewiki --fraction 0.5 --epochs 3 --no-base --group-cols --batch-f 256 --out gpurun_out/scale_hugewiki_half_grouped256.json > gpurun_out/r02q_g256.log 2>&1
python tools/scale_emulation.py --workload netflix --epochs 3 --out gpurun_out/scale_netflix_plain.json > gpurun_out/r02q_nplain.log 2>&1
python tools/scale_emulation.py --workload netflix --epochs 3 --no-base --group-cols --batch-f 1024 --out gpurun_out/scale_netflix_grouped1024.json > gpurun_out/r02q_ng1024.log 2>&1

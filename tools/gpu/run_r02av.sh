# configs[2] at HEAD: Yahoo!Music-shaped batch-Hogwild vs deterministic wavefront
python tools/sweep.py --name r02av_yahoo --set yahoo3 --steps 6 --warmup 3 > gpurun_out/r02av.log 2>&1
cat gpurun_out/r02av_yahoo.md

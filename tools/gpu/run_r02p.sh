set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv
python -m pytest tests -m gpu -q --timeout 2400 -p no:cacheprovider > gpurun_out/r02p_gputests.log 2>&1
tail -5 gpurun_out/r02p_gputests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02p_smoke.log 2>&1
python bench.py > gpurun_out/r02p_bench.log 2>&1
B="python bench.py --steps 1 --warmup 2 --no-e2e --no-cpu-baseline --no-deterministic"
ncu --set full --clock-control none --import-source on -k regex:k_hogwild -s 2 -c 1 -o /tmp/r02p_hog -f $B > /dev/null 2>&1
ncu -i /tmp/r02p_hog.ncu-rep --page raw --csv > gpurun_out/r02p_hog_raw.csv
ncu --set full --clock-control none -k regex:k_hogwild -s 2 -c 1 -o /tmp/r02p_hogg -f $B --group-cols --batch-f 1024 > /dev/null 2>&1
ncu -i /tmp/r02p_hogg.ncu-rep --page raw --csv > gpurun_out/r02p_hog_grouped_raw.csv
ncu --set full --clock-control none -k regex:k_wavefront2 -s 1 -c 1 -o /tmp/r02p_wf -f $B --schedule wavefront --storage fp32 --workers 888 --wf-cols 7680 --cyclic > /dev/null 2>&1
ncu -i /tmp/r02p_wf.ncu-rep --page raw --csv > gpurun_out/r02p_wf_raw.csv
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02p_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
S="python bench.py --steps 5 --warmup 2 --no-cpu-baseline --no-e2e --no-deterministic --grid-a 8"
$S > gpurun_out/r02p_a8_resident.log 2>&1
$S --staged 1 > gpurun_out/r02p_a8_staged1.log 2>&1
$S --staged 2 > gpurun_out/r02p_a8_staged2.log 2>&1
python bench.py --workload hugewiki --steps 3 --warmup 2 > gpurun_out/r02p_hugewiki.log 2>&1
ls -la gpurun_out

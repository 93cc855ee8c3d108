# deterministic wavefront fp16 k = 128: s / c sweep around the fp32 optimum (s = 888, c = 7680)
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic --schedule wavefront --storage fp16 --cyclic --steps 4 --warmup 2"
for sc in "888 6144" "888 7680" "888 9216" "888 10240" "840 7680" "768 7680" "888 12288"; do set -- $sc
  $B --workers $1 --wf-cols $2 2>/dev/null | tail -n 1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('s=$1 c=$2', round(d['ms_per_step'],3), round(d['roofline']['sgd_ms_per_epoch'],3), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])"
done

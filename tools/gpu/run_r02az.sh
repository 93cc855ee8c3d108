# A/B: k_wavefront2 register cap: __launch_bounds__(128) (ptxas picks 96 for fp16 with a 24-B spill) vs __maxnreg__(128 / 168)
B="python bench.py --no-e2e --no-cpu-baseline --no-deterministic --schedule wavefront --workers 888 --wf-cols 7680 --cyclic --steps 4 --warmup 2"
for v in base wf128 wf168; do
  if [ $v = base ]; then unset MF_LIB; else export MF_LIB=tools/bin/$v.so; fi
  for s in fp16 fp32 bf16; do
    $B --storage $s 2>/dev/null | tail -n 1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v $s', round(d['ms_per_step'],3), round(d['roofline']['sgd_ms_per_epoch'],3), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])"
  done
  $B --storage fp16 --k 64 2>/dev/null | tail -n 1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v fp16 k64', round(d['ms_per_step'],3), round(d['roofline']['sgd_ms_per_epoch'],3), round(d['roofline']['frac'],3))"
done

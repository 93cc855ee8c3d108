# resident Hogwild blocks per SM: 5 (48 regs, HEAD) vs 6 (40 regs, spills) vs 8 (32 regs, spills)
for v in base tools/bin/minb6.so tools/bin/minb8.so; do
  if [ $v = base ]; then unset MF_LIB; else export MF_LIB=$v; fi
  for w in "--workload netflix" "--workload yahoo" "--workload hugewiki --steps 3 --warmup 3" "--workload hugewiki --steps 3 --warmup 3 --group-cols --batch-f 4096"; do
    python bench.py --no-e2e --no-cpu-baseline --no-deterministic --steps 10 $w 2>&1 | grep "^{" | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', '$w', round(d['ms_per_step'],3), d['roofline']['workers'], d['clocks']['sm_mhz'])"
  done
done

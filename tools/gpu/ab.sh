# usage: bash tools/gpu/ab.sh <variant.so> [bench args...]: base vs variant, netflix + yahoo + k32
V=$1; shift
for v in base $V; do for w in "--workload netflix" "--workload yahoo" "--workload netflix --k 32"; do
  if [ $v = base ]; then unset MF_LIB; else export MF_LIB=$v; fi
  python bench.py --no-e2e --no-cpu-baseline --no-deterministic --steps 10 $w "$@" 2>&1 | grep "^{" | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', '$w', round(d['ms_per_step'],3))"
done; done

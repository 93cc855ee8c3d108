# round-2 verification: full GPU suite, smoke, default bench line, reference arm
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
python -m pytest tests -m gpu -q --timeout 1800 -p no:cacheprovider > gpurun_out/r02ab_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r02ab_tests.log
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > gpurun_out/r02ab_smoke.log 2>&1
python bench.py > gpurun_out/r02ab_bench.log 2>&1
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r02ab_ref.log 2>&1
tail -3 gpurun_out/r02ab_tests.log; tail -1 gpurun_out/r02ab_smoke.log

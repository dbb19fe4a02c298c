#!/bin/bash
# session s14: mu-sweep L1 experiments (own cd_x by shuffles, L1 load
# policies) as same-box A/B rounds at 256^3, after the corner parity tests
OUT=gpurun_out/${1:-r02s14}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py -q -k "corners or rejects" > $OUT/pytest_corners.log 2>&1; echo "exit $?" >> $OUT/pytest_corners.log
for i in 1 2; do
  for t in '{}' '{"mu_xshfl": 1}' '{"mu_ldhint": 1}' '{"mu_ldhint": 2}' '{"mu_ldhint": 3}' '{"mu_xshfl": 1, "mu_ldhint": 3}' '{"mu_xshfl": 1, "mu_ldhint": 2}'; do
    echo "$t" >> $OUT/ab.jsonl
    timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 --tuning "$t" >> $OUT/ab.jsonl 2>> $OUT/bench.err
  done
done
echo done > $OUT/DONE

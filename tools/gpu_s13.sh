#!/bin/bash
# session s13: the carried halo ring (mu_hcar): corner parity / bitwise,
# sanitizer over every kernel family, A/B pairs of the mu-sweep at 256^3
OUT=gpurun_out/${1:-r02s13}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py -q -k "corners or rejects" > $OUT/pytest_corners.log 2>&1; echo "exit $?" >> $OUT/pytest_corners.log
for i in 1 2 3; do
  for t in '{"mu_hcar": 0}' '{"mu_hcar": 1}' '{"mu_hcar": 1, "mu_halo_l1": 0}'; do
    echo "$t" >> $OUT/ab.jsonl
    timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 --tuning "$t" >> $OUT/ab.jsonl 2>> $OUT/bench.err
  done
done
timeout 1500 python -m pytest tests/test_gpu_aux.py -q -k sanitizer > $OUT/pytest_sanitizer.log 2>&1; echo "exit $?" >> $OUT/pytest_sanitizer.log
echo done > $OUT/DONE

#!/bin/bash
# session s18: P2 phi without the 2/sc division (select), parity + timing
OUT=gpurun_out/${1:-r02s18}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_p2.py -m gpu -q -x > $OUT/pytest_p2.log 2>&1; echo "exit $?" >> $OUT/pytest_p2.log
for i in 1 2; do
  for cfg in "PF_P2_MINB=4" "PF_P2_MINB=3"; do
    echo "$cfg" >> $OUT/ab.jsonl
    env $cfg timeout 600 python bench.py --steps 40 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --autotune 0 >> $OUT/ab.jsonl 2>> $OUT/bench.err
  done
done
echo done > $OUT/DONE

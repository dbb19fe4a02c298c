#!/bin/bash
# session s20: P2 side-staged tilings (PF_P2_SIDE) + P2 multi-block bitwise
OUT=gpurun_out/${1:-r02s20}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_p2.py -m gpu -q -x > $OUT/pytest_p2.log 2>&1; echo "exit $?" >> $OUT/pytest_p2.log
timeout 1200 python -m pytest tests/test_gpu_multiblock.py -m gpu -q -x -k p2 > $OUT/pytest_mb_p2.log 2>&1; echo "exit $?" >> $OUT/pytest_mb_p2.log
for i in 1 2; do
  for cfg in "PF_P2_SIDE=8x2" "PF_P2_SIDE=8x1" "PF_P2_SIDE=4x3" "PF_P2_SIDE=4x4"; do
    echo "$cfg" >> $OUT/ab.jsonl
    env $cfg timeout 600 python bench.py --steps 40 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --autotune 0 >> $OUT/ab.jsonl 2>> $OUT/bench.err
  done
done
echo done > $OUT/DONE

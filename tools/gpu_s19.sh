#!/bin/bash
# session s19: P2 side-staged phi kernel -- parity, A/B against z-marching phi
OUT=gpurun_out/${1:-r02s19}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_p2.py -m gpu -q -x > $OUT/pytest_p2.log 2>&1; echo "exit $?" >> $OUT/pytest_p2.log
for i in 1 2; do
  for cfg in "PF_P2_PHI=march" "PF_P2_PHI=side" "PF_P2_PHI=side PF_P2_SIDE_PD=0" "PF_P2_PHI=side PF_P2_SIDE_PD=3"; do
    echo "$cfg" >> $OUT/ab.jsonl
    env $cfg timeout 600 python bench.py --steps 40 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --autotune 0 >> $OUT/ab.jsonl 2>> $OUT/bench.err
  done
done
echo done > $OUT/DONE

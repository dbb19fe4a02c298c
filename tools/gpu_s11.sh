#!/bin/bash
# session r02 s11: P2 A/B (occupancy, L2 prefetch) + P2 parity
OUT=gpurun_out/r02s11
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
PF_P2_MINB=4 timeout 900 python -m pytest tests/test_gpu_p2.py -m gpu -q -x > $OUT/pytest_minb4.log 2>&1; echo "exit $?" >> $OUT/pytest_minb4.log
timeout 900 python -m pytest tests/test_gpu_p2.py -m gpu -q -x > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
i=0
for cfg in "-" "PF_P2_MINB=4" "PF_P2_PREFETCH=0" "PF_P2_MINB=4 PF_P2_PREFETCH=0" "-" "PF_P2_MINB=4"; do
  i=$((i+1)); echo "$i: $cfg" >> $OUT/configs.txt
  e=$cfg; [ "$e" == "-" ] && e=""
  env $e timeout 600 python bench.py --steps 40 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --autotune 0 > $OUT/bench_$i.json 2>> $OUT/bench.err
done
echo done > $OUT/DONE

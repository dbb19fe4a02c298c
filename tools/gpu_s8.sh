#!/bin/bash
OUT=gpurun_out/r02s8
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_p2.py -m gpu -q > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
timeout 600 python bench.py --steps 40 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --autotune 0 > $OUT/bench.json 2> $OUT/bench.err
PF_P2_NAIVE=1 timeout 600 python bench.py --steps 40 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --autotune 0 > $OUT/bench_naive.json 2>> $OUT/bench.err
echo done > $OUT/DONE

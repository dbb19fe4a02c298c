#!/bin/bash
# session s26: P2 tuning knobs + P2 autotune; P2 suite and P2 bench line
OUT=gpurun_out/${1:-r02s26}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_p2.py tests/test_gpu_autotune.py -m gpu -q -x > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
timeout 900 python bench.py --steps 40 --warmup 5 --no-cpu-baseline --no-e2e --no-stress > $OUT/bench.json 2>> $OUT/bench.err
echo done > $OUT/DONE

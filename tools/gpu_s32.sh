#!/bin/bash
# session s32: P2 specialisation with compile-time geometry and folded zero / unit coefficients, 4x5 / 4x6 tiles
OUT=gpurun_out/${1:-r02s32}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_p2.py -m gpu -q -x > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
timeout 900 python bench.py --steps 40 --warmup 5 --no-cpu-baseline --no-e2e --no-stress > $OUT/bench.json 2>> $OUT/bench.err
echo done > $OUT/DONE

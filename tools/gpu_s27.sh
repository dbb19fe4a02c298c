#!/bin/bash
# session s27: anti-trapping skip (mu_atskip) -- corners bitwise / parity, bench line
OUT=gpurun_out/${1:-r02s27}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py -q -k "corners" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
timeout 900 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --no-stress --no-p2 --autotune 0 > $OUT/bench.json 2>> $OUT/bench.err
echo done > $OUT/DONE

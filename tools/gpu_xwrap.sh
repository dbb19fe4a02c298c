#!/bin/bash
# GPU parity suite + A/B of the x-wrap (no x ghost columns) against PF_NO_XWRAP=1
TAG=${1:-xw}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu.log
for r in 1 2; do
timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --autotune 0 > $OUT/bench_xw_$r.json 2>> $OUT/bench.err
PF_NO_XWRAP=1 timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --autotune 0 > $OUT/bench_noxw_$r.json 2>> $OUT/bench.err
done
echo done > $OUT/DONE

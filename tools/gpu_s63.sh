#!/bin/bash
# session s63: stress-set line with two auto-tuning passes
OUT=gpurun_out/${1:-r02s63}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --no-p2 > $OUT/bench.json 2> $OUT/bench.err
echo done > $OUT/DONE

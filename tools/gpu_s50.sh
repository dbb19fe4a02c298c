#!/bin/bash
# session s50: D.8 data independence with the final kernels (+ the atskip variant per IC)
OUT=gpurun_out/${1:-r02s50}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python tools/ic_independence.py > $OUT/ic_independence.json 2> $OUT/ic.err
echo done > $OUT/DONE

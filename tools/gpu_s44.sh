#!/bin/bash
# session s44: config 5 (400x400x2000 DS, 20k steps) with the final kernels
OUT=gpurun_out/${1:-r02s44}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1500 python tools/config5.py --out $OUT/config5.jsonl > $OUT/config5.log 2>&1
echo done > $OUT/DONE

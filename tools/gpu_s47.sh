#!/bin/bash
# session s47: mu_zbal (lower row's z-face before the first barrier in warps < zbal) -- corners + A/B
OUT=gpurun_out/${1:-r02s47}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py -q -x -k "corner" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
bash tools/gpu_ab_pairs.sh r02s47ab 2 '{}' '{"mu_zbal": 1}' '{"mu_zbal": 2}'
echo done > $OUT/DONE

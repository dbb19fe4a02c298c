#!/bin/bash
# session s56: mu_xring (edge lanes' outer x-neighbour from the staged ring) -- corners + A/B
OUT=gpurun_out/${1:-r02s56}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py -q -x -k "corner" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
bash tools/gpu_ab_pairs.sh r02s56ab 3 '{}' '{"mu_xring": 1}'
echo done > $OUT/DONE

#!/bin/bash
# session s40: mu_hasync 3 (own phi_dst / mu staged too) -- bitwise corners + A/B pairs
OUT=gpurun_out/${1:-r02s40}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py -q -x -k "corner" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
bash tools/gpu_ab_pairs.sh r02s40ab 2 '{}' '{"mu_hasync": 3}'
echo done > $OUT/DONE

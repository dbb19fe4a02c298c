#!/bin/bash
# session s58: phi_prefetch 3 (only the cells' mu lines into L2) -- corners + A/B
OUT=gpurun_out/${1:-r02s58}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py -q -x -k "corner" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
bash tools/gpu_ab_pairs.sh r02s58ab 2 '{}' '{"phi_prefetch": 3, "phi_pfd": 1}' '{"phi_prefetch": 3, "phi_pfd": 2}' '{"phi_prefetch": 3, "phi_pfd": 3}' '{"phi_prefetch": 3, "phi_pfd": 4}'
echo done > $OUT/DONE

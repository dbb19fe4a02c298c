#!/bin/bash
# session s52: mu_zrev (mu z-chunks top down, phi_dst still in L2) -- corners + A/B
OUT=gpurun_out/${1:-r02s52}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py -q -x -k "corner" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
bash tools/gpu_ab_pairs.sh r02s52ab 3 '{}' '{"mu_zrev": 1}'
echo done > $OUT/DONE

#!/bin/bash
# session s36: mu_hasync 1..3 -- bitwise corners + A/B pairs
OUT=gpurun_out/${1:-r02s36}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py -q -x -k "corner" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
bash tools/gpu_ab_pairs.sh r02s36ab 2 '{}' '{"mu_hasync": 1, "mu_halo_l1": 0}' '{"mu_hasync": 2, "mu_halo_l1": 0}' '{"mu_hasync": 3, "mu_halo_l1": 0}' '{"mu_hasync": 3}'
echo done > $OUT/DONE

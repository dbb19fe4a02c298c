#!/bin/bash
# session s39: mu_hasync 2 (whole halo tile's phi_src staged) -- bitwise corners + A/B pairs
OUT=gpurun_out/${1:-r02s39}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py -q -x -k "corner" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
bash tools/gpu_ab_pairs.sh r02s39ab 2 '{}' '{"mu_hasync": 2}' '{"mu_hasync": 2, "mu_zc": 16}' '{"mu_hasync": 2, "mu_pfd": 3}'
echo done > $OUT/DONE

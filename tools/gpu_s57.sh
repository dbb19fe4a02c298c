#!/bin/bash
# session s57: phi_muearly (the phi-sweep's mu loads before the faces / one plane ahead) -- corners + A/B
OUT=gpurun_out/${1:-r02s57}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py -q -x -k "corner" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
bash tools/gpu_ab_pairs.sh r02s57ab 2 '{}' '{"phi_muearly": 1}' '{"phi_muearly": 2}' '{"phi_muearly": 2, "phi_minb": 4}' '{"phi_muearly": 1, "phi_minb": 4}'
echo done > $OUT/DONE

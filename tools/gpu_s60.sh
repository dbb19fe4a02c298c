#!/bin/bash
# session s60: the new full-size tests (stress set sampled cells, tunings bitwise at the bench configuration)
OUT=gpurun_out/${1:-r02s60}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -m gpu -q > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
echo done > $OUT/DONE

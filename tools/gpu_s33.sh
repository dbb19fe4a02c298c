#!/bin/bash
OUT=gpurun_out/${1:-r02s33}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for o in ""; do
  PF_NVRTC_OPTS="$o" STEPS=1 timeout 300 python tools/p2_bitwise_probe.py >> $OUT/probe.log 2>&1
done
timeout 1500 python -m pytest tests/test_gpu_p2.py -m gpu -q -x > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
echo done > $OUT/DONE

#!/bin/bash
# session s53: P2 DS recipe -- P2 tests + bench P2 line with the DS sub-line
OUT=gpurun_out/${1:-r02s53}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_p2.py -m gpu -q -x > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
timeout 900 python bench.py --steps 40 --warmup 5 --no-cpu-baseline --no-e2e --no-stress > $OUT/bench.json 2> $OUT/bench.err
echo done > $OUT/DONE

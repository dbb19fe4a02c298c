#!/bin/bash
# session s45: concurrent slab schedule (sched 2) -- bitwise tests + A/B
OUT=gpurun_out/${1:-r02s45}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py -q -x -k "slab or step_schedule" > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
bash tools/gpu_ab_pairs.sh r02s45ab 2 '{}' '{"sched": 2, "slab": 1}' '{"sched": 2, "slab": 2}' '{"sched": 2, "slab": 4}' '{"sched": 1, "slab": 2}'
echo done > $OUT/DONE

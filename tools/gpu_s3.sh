#!/bin/bash
# session r02 s3: full GPU suite (incl. multi-block), layout A/B, long DS tuning
OUT=gpurun_out/r02s3
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > $OUT/pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/pytest_gpu.log
bash tools/gpu_ab_env.sh r02s3/ab - PF_LAYOUT=soa - PF_LAYOUT=soa
timeout 900 python tools/ds_tune.py --steps 20000 --check 2000 --vs 0.05,0.1 --Gs 0.05 --zf 0.49 > $OUT/ds_tune.jsonl 2> $OUT/ds_tune.err
echo done > $OUT/DONE

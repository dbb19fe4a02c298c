#!/bin/bash
# session r02 s2: A/B of mu-sweep variants + DS workload tuning + parity of the changed kernels
OUT=gpurun_out/r02s2
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > $OUT/pytest_parity.log 2>&1; echo "exit $?" >> $OUT/pytest_parity.log
bash tools/gpu_ab_env.sh r02s2/ab - PF_NO_MSOL=1 "PF_NVRTC_OPTS=-DPF_MU_UNROLL=2" - PF_NO_MSOL=1 "PF_NVRTC_OPTS=-DPF_MU_UNROLL=2"
timeout 600 python tools/ds_tune.py --steps 4000 --check 500 > $OUT/ds_tune.jsonl 2> $OUT/ds_tune.err
echo done > $OUT/DONE

#!/bin/bash
# session r02 s5: persistent-launch A/B, TMA/TMEM probes, autotune+aux tests
OUT=gpurun_out/r02s5
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 60 tools/build/tma_probe2 > $OUT/tma_probe2.json 2>&1; echo "exit $?" >> $OUT/tma_probe2.json
timeout 60 tools/build/tmem_probe > $OUT/tmem_probe.json 2>&1; echo "exit $?" >> $OUT/tmem_probe.json
timeout 900 python -m pytest tests/test_gpu_autotune.py tests/test_gpu_aux.py -m gpu -q -x > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
bash tools/gpu_ab_env.sh r02s5/ab - PF_MU_PERS=1 PF_PHI_PERS=1 "PF_MU_PERS=1 PF_PHI_PERS=1" - PF_MU_PERS=1 PF_PHI_PERS=1
echo done > $OUT/DONE

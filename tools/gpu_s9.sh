#!/bin/bash
# session r02 s9: TMEM mu-sweep A/B + parity; P2 parity after the rcp/rsqrt change
OUT=gpurun_out/r02s9
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_autotune.py tests/test_gpu_p2.py -m gpu -q -x > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
bash tools/gpu_ab_env.sh r02s9/ab - "PF_MU_TMEM=1 PF_MU_RPF=0" "PF_MU_TMEM=1 PF_MU_RPF=0 PF_MU_MINB=3" "PF_MU_RPF=0 PF_MU_MINB=3" "PF_MU_TMEM=1 PF_MU_MINB=3" - "PF_MU_TMEM=1 PF_MU_RPF=0 PF_MU_MINB=3"
echo done > $OUT/DONE

#!/bin/bash
# session s41: P2 mu halo ring staged by cp.async (p2_mu_hasync) -- P2 tests, A/B
OUT=gpurun_out/${1:-r02s41}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_p2.py -m gpu -q -x > $OUT/pytest.log 2>&1; echo "exit $?" >> $OUT/pytest.log
for r in 1 2; do
  timeout 600 python tools/p2_ab.py '{"p2_phi": 1, "p2_mu_hasync": 0}' '{"p2_phi": 1}' '{"p2_phi": 1, "p2_mu_ty": 4, "p2_mu_minb": 3}' '{"p2_phi": 1, "p2_mu_ty": 4, "p2_mu_minb": 5}' >> $OUT/p2_ab.jsonl 2>> $OUT/p2_ab.err
done
echo done > $OUT/DONE

#!/bin/bash
# session s16: ncu --set full of the P2 kernels (side-staged mu, z-marching phi)
OUT=gpurun_out/${1:-r02s16}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_mu_side -s 2 -c 1 -o $OUT/prof_p2mu \
   python tools/p2_run.py 256 4 > $OUT/ncu_p2mu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_phi_march -s 2 -c 1 -o $OUT/prof_p2phi \
   python tools/p2_run.py 256 4 > $OUT/ncu_p2phi.log 2>&1
echo done > $OUT/DONE

mkdir -p gpurun_out
cp tools/reorder_round_profile.py build/r02a/tools/
(cd build/r02a && timeout 600 python tools/reorder_round_profile.py > ../../gpurun_out/ab14_r02a.txt 2>&1)
timeout 600 python tools/reorder_round_profile.py > gpurun_out/ab14_head.txt 2>&1

python tools/build.py > /dev/null
mkdir -p gpurun_out
timeout 600 python tools/scratch/reorder_probe.py > gpurun_out/reorder_probe_r02f.txt 2>&1
timeout 300 python tools/c1_latency.py > gpurun_out/c1_r02f.txt 2>&1

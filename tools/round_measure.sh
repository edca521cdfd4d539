#!/bin/bash
# Full measurement pass for a round (run on the GPU box): bench (default settings),
# reference arm, ncu launch list and --set full captures of the hot kernels.
set -u
TAG=${TAG:-r01}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_gpu.txt 2>&1
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${TAG}_reference.json 2>&1
LAUNCHES=1 WARM=1 TAG=$TAG KERNELS="${KERNELS:-k1p_fwd k2t_fwd k3t_pair k4p_pair k5_ccf}" bash tools/ncu_profile.sh > /dev/null 2>&1
ls -la gpurun_out | tail -30

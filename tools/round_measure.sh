#!/bin/bash
# Full measurement pass for a round (run on the GPU box): bench (default settings),
# reference arm, ncu launch list and --set full captures of the hot kernels, summarised on
# the box (the .ncu-rep files are large; only the dominant kernel's report is kept).
set -u
TAG=${TAG:-r01}
KEEP=${KEEP:-k3t_pair}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_gpu.txt 2>&1
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${TAG}_reference.json 2>&1
KS="${KERNELS:-k1p_fwd k2t_fwd k3t_pair k4p_pair k5_ccf}"
LAUNCHES=1 WARM=1 TAG=$TAG KERNELS="$KS" bash tools/ncu_profile.sh > /dev/null 2>&1
python tools/launch_shares.py gpurun_out/${TAG}_launches.csv > gpurun_out/${TAG}_launch_shares.txt 2>&1
for k in $KS; do
  python tools/ncu_summary.py gpurun_out/${TAG}_${k}.ncu-rep gpurun_out/${TAG}_${k}_warm.ncu-rep \
      > gpurun_out/${TAG}_ncu_${k}.txt 2>&1
done
python tools/ncu_traffic.py $TAG $KS > gpurun_out/${TAG}_ncu_traffic.json 2> gpurun_out/${TAG}_ncu_traffic.err
for k in $KS; do
  [ "$k" = "$KEEP" ] || rm -f gpurun_out/${TAG}_${k}.ncu-rep
  rm -f gpurun_out/${TAG}_${k}_warm.ncu-rep
done
du -sh gpurun_out; ls gpurun_out

#!/bin/bash
# Full measurement pass for a round (run on the GPU box through gpurun): the bench line (default
# settings), the reference arm, the fp64 / bounded-pool / time-series lines, the ncu launch list,
# `--set full` captures of the hot kernels (cold and warm L2) summarised on the box, the DRAM
# traffic JSON the bench line reads (profiles/ncu_traffic.json), compute-sanitizer.
# Only the dominant kernel's .ncu-rep is kept (the files are large).
set -u
TAG=${TAG:-r02}
KEEP=${KEEP:-k3t_pair}
KS="${KERNELS:-k1w_fwd k2t_fwd k3t_pair k4w_pair k5_ccf}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_gpu.txt 2>&1
nproc >> gpurun_out/${TAG}_gpu.txt; lscpu | grep -E "Model name|Socket" >> gpurun_out/${TAG}_gpu.txt
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${TAG}_reference.json 2>&1
timeout 900 python bench.py --precision f64 --steps 5 --warmup 2 --no-cpu-baseline > gpurun_out/${TAG}_f64.json 2>&1
timeout 900 python bench.py --pool 160 --steps 5 --warmup 2 --no-cpu-baseline > gpurun_out/${TAG}_pool.json 2>&1
timeout 900 python bench.py --config 4 --ts-grids 24 --warmup 2 > gpurun_out/${TAG}_config4.json 2>&1
timeout 900 python bench.py --config 2 --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/${TAG}_config2.json 2>&1
timeout 900 python bench.py --compose --steps 5 --warmup 2 --no-cpu-baseline > gpurun_out/${TAG}_compose.json 2>&1
timeout 900 python bench.py --config 5 --steps 5 --warmup 2 --no-cpu-baseline --e2e-steps 1 > gpurun_out/${TAG}_config5.json 2>&1
timeout 900 python bench.py --config 5 --pool 480 --steps 3 --warmup 1 --no-cpu-baseline --e2e-steps 1 > gpurun_out/${TAG}_config5_pool.json 2>&1
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
timeout 1500 bash tools/sanitize.sh > gpurun_out/${TAG}_sanitize.txt 2>&1
du -sh gpurun_out; ls gpurun_out | grep "^${TAG}_"

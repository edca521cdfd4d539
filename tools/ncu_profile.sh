#!/bin/bash
# Profile one bench step under ncu (run on the GPU box via gpurun; 1 GPU).
#   1) launch list with per-launch device time (cold-cache, serialised: compare shares)
#   2) one `--set full` capture of each hot kernel (K1..K5)
# Outputs land in gpurun_out/ (scratch); summaries are copied into profiles/ by hand.
set -u
OUT=${OUT:-gpurun_out}
TAG=${TAG:-r01}
KERNELS=${KERNELS:-"k1_fwd_rows k2_fwd_cols k3_pair_cols k4_pair_rows k5_ccf_moments"}
BENCH="python bench.py --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 1"
mkdir -p "$OUT"
if [ "${LAUNCHES:-1}" = 1 ]; then
  ncu --metrics gpu__time_duration.sum --clock-control none -c ${NLAUNCH:-1900} --csv \
      --log-file "$OUT/${TAG}_launches.csv" $BENCH > "$OUT/${TAG}_launches_bench.log" 2>&1
fi
for k in $KERNELS; do
  skip=${SKIP:-4}
  case $k in k5*|k6*) skip=0;; esac
  ncu --set full --clock-control none --import-source on -k regex:$k -s $skip -c 1 \
      -o "$OUT/${TAG}_$k" -f $BENCH > "$OUT/${TAG}_$k.log" 2>&1
  if [ "${WARM:-0}" = 1 ]; then   # warm-L2 variant: no cache flush between replays
    ncu --set full --cache-control none --clock-control none -k regex:$k -s $skip -c 1 \
        -o "$OUT/${TAG}_${k}_warm" -f $BENCH > "$OUT/${TAG}_${k}_warm.log" 2>&1
  fi
done
ls -la "$OUT"

#!/bin/bash
# Bench sweep over chunk sizes (device-timed value only), one JSON summary line each.
for cp in ${CPS:-8 16 32}; do
  for ct in ${CTS:-8}; do
    timeout 600 python bench.py --chunk-pairs $cp --chunk-tiles $ct --no-cpu-baseline --e2e-steps 1 \
      ${EXTRA:-} 2>&1 | tail -1 | python tools/bench_brief.py "cp=$cp ct=$ct"
  done
done

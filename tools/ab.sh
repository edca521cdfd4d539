#!/bin/bash
# Interleaved same-box A/B of two builds of the library (abtmp/A.so, abtmp/B.so): bench.py's
# device-timed step and per-kernel times, REPS repetitions each.
L=paper_conf_icpp_blattnerkcsbz14_b200/libstitch_b200.so
for r in $(seq ${REPS:-2}); do
  for v in ${VARIANTS:-A B}; do
    cp abtmp/$v.so $L
    timeout 600 python bench.py --no-cpu-baseline --e2e-steps 1 ${EXTRA:-} 2>/dev/null | tail -1 | python tools/bench_brief.py "$v$r"
  done
done

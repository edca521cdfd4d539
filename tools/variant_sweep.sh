#!/bin/bash
# A/B several prebuilt library variants (variants/*.so) with the same bench settings.
PKG=paper_conf_icpp_blattnerkcsbz14_b200
cp $PKG/libstitch_b200.so /tmp/lib_orig.so
for v in ${VARIANTS:-variants/*.so}; do
  cp $v $PKG/libstitch_b200.so
  CPS=${CPS:-24} CTS=${CTS:-16} bash tools/bench_sweep.sh 2>&1 | sed "s|^|$(basename $v) |"
done
cp /tmp/lib_orig.so $PKG/libstitch_b200.so

#!/bin/bash
# A/B of library BUILDS on one probe:  tools/ab_libs.sh OUT lib1.so lib2.so ... -- probe args
# each lib is copied over paper_conf_ipps_dieguezadnm18_b200/libscanb200.so before the probe
out=$1; shift
libs=()
while [ "$1" != "--" ]; do libs+=("$1"); shift; done
shift
dst=paper_conf_ipps_dieguezadnm18_b200/libscanb200.so
cp $dst /tmp/libscanb200.orig.so
for l in "${libs[@]}"; do
  echo "### lib: $l" >> "$out"
  cp "$l" $dst
  python "$@" >> "$out" 2>&1
done
cp /tmp/libscanb200.orig.so $dst

#!/bin/bash
# mk_ab.sh NAME "DEFS": copy the working tree (tracked + untracked, not ignored) to ab_NAME/, copy the
# built helper libraries, and build libwg.so there with WG_NVCC_DEFS=DEFS (A/B variant for ab_multi.sh).
set -e
n=$1
defs=$2
rm -rf "ab_$n"
mkdir "ab_$n"
git ls-files -co --exclude-standard | grep -v '^ab_' | tar -cf - -T - | tar -xf - -C "ab_$n"
cp synth/libwggen.so synth/libwggen_host.so "ab_$n/synth/"
cp oracle/liboracle.so "ab_$n/oracle/"
[ -f MEASURED_PEAKS.json ] && cp MEASURED_PEAKS.json "ab_$n/"
(cd "ab_$n" && WG_NVCC_DEFS="$defs" python -c "from paper_conf_sc_yanglql22_b200._build import build_lib; build_lib(force=True)")
echo "ab_$n built with WG_NVCC_DEFS='$defs'"

#!/bin/bash
# mk_ab_rev.sh NAME REV: ab_NAME/ = the tree of git revision REV (helper libraries copied, libwg.so built),
# for ab_multi.sh A/Bs of the working tree against a committed state.
set -e
n=$1
rev=$2
rm -rf "ab_$n"
mkdir "ab_$n"
git archive "$rev" | tar -x -C "ab_$n"
cp synth/libwggen.so synth/libwggen_host.so "ab_$n/synth/"
cp oracle/liboracle.so "ab_$n/oracle/"
[ -f MEASURED_PEAKS.json ] && cp MEASURED_PEAKS.json "ab_$n/"
(cd "ab_$n" && python -c "from paper_conf_sc_yanglql22_b200._build import build_lib; build_lib(force=True)")
echo "ab_$n = $rev"

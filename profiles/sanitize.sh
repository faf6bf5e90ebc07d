#!/bin/bash
# compute-sanitizer pass over libwg.so (SURVEY.md section 4 tier 4): the four tools on the tiny-config
# workload of profiles/sanitize_run.py, restricted to this library's kernels (mangled names contain "2wg";
# initcheck instruments every kernel, see below).
# Logs: gpurun_out/sanitize_<tool>.log (copied to profiles/<round>/ when judged).
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
python profiles/sanitize_run.py > gpurun_out/sanitize_plain.log 2>&1; echo "plain rc=$?"; tail -1 gpurun_out/sanitize_plain.log
for tool in memcheck racecheck synccheck initcheck; do
  extra=""
  [ $tool = memcheck ] && extra="--leak-check no --padding 32"
  [ $tool = racecheck ] && extra="--racecheck-report all"
  # initcheck tracks initialisation only through the kernels it instruments: with the wg filter, buffers
  # torch fills (ones_like, zeros) would read as uninitialised, so initcheck instruments every kernel
  filt="--kernel-name kns=2wg"
  [ $tool = initcheck ] && filt=""
  timeout ${SAN_TIMEOUT:-1500} $CS --tool $tool $extra $filt --print-limit 200 \
      --error-exitcode 17 python profiles/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|SANITIZE WORKLOAD OK" gpurun_out/sanitize_$tool.log | tail -3
done

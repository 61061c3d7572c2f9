#!/bin/bash
# Development probe: repeat one sanitizer run of tests/sanitize_target.py and
# keep the output of any run that does not exit within 60 s (the rare hang at
# process exit under compute-sanitizer).  Usage: tools/san_exit_probe.sh TOOL GROUP N
tool=$1; group=$2; n=$3
mkdir -p gpurun_out
for i in $(seq 1 $n); do
  SLATE_EXIT_TRACE=1 SLATE_STANDBY_TIMEOUT_US=20000 SANITIZE_FAST_EXIT=${FAST:-1} timeout -s KILL 60 compute-sanitizer --tool $tool --error-exitcode 97 \
    python tests/sanitize_target.py $group > gpurun_out/sanx_$i.log 2>&1
  rc=$?
  echo "run $i rc=$rc $(grep -c 'ERROR SUMMARY: 0 errors' gpurun_out/sanx_$i.log)" >> gpurun_out/sanx_summary.log
  if [ $rc -ne 137 ]; then rm -f gpurun_out/sanx_$i.log; fi
done

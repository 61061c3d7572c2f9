#!/bin/bash
# One GPU call that refreshes the C2 (headline) artefacts under gpurun_out/:
# the bench line; the kernel launch list of the bench's TIMED region (ncu,
# NVTX range "timed", cold-cache serialised replay); an ncu --set full
# capture of the C2 tenants' workers and original kernels.  Run from the repo
# root under gpurun; summaries are copied into profiles/ afterwards.
set -u
timeout 900 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
SLATE_NVTX=1 timeout 1200 ncu --nvtx --nvtx-include "timed/" --metrics gpu__time_duration.sum --clock-control none \
  -c 5000 --csv --log-file gpurun_out/launches_c2.csv \
  python bench.py --steps 2 --warmup 3 --no-c3 --no-c4 --no-cpu-baseline > gpurun_out/launches_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:slate_worker|spmv_worker|standalone" -c 8 \
  -o gpurun_out/prof_c2 python tools/ncu_target.py 1 > gpurun_out/prof_c2.log 2>&1
ls -la gpurun_out | tail -20

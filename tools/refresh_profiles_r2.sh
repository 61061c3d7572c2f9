#!/bin/bash
# One GPU call that refreshes the round-2 artefacts under gpurun_out/: the bench
# line; the kernel launch list of the bench's TIMED region (ncu, NVTX range
# "timed", cold-cache serialised replay); an ncu --set full capture of the
# C2 / C4 tenants (tools/ncu_target_r2.py).  Run from the repo root under
# gpurun; summaries are copied into profiles/ afterwards (tools/ncu_summary.py,
# tools/launch_list.py).
set -u
timeout 1500 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_r2.json 2> gpurun_out/bench_r2.err
SLATE_NVTX=1 timeout 1200 ncu --nvtx --nvtx-include "timed/" --metrics gpu__time_duration.sum --clock-control none \
  -c 5000 --csv --log-file gpurun_out/launches_c2_r2.csv \
  python bench.py --steps 2 --warmup 3 --no-c3 --no-c4 --no-cpu-baseline > gpurun_out/launches_c2_r2.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on \
  -k "regex:spmv_worker|slate_worker|standalone" -o gpurun_out/prof_r2 --force-overwrite \
  python tools/ncu_target_r2.py > gpurun_out/prof_r2.log 2>&1
ls -la gpurun_out | tail -20

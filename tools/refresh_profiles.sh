#!/bin/bash
# One GPU call that refreshes every measured artefact under gpurun_out/ (copied
# into profiles/ afterwards, here): bench line, C3 split sweep, C3 interference
# diagnostics, the bench's kernel launch list and ncu --set full captures of
# the C2 and C3 tenants.  Run from the repo root under gpurun.
set -u
timeout 900 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err
SLATE_SWEEP_SPLITS=40,48,56,60,64,68,72,76,80 SLATE_C3_REPS=1 SLATE_SWEEP_OUT=gpurun_out/c3_sweep_r1.json \
  timeout 300 python tools/c3_sweep.py > gpurun_out/c3_sweep_r1.txt 2>&1
SLATE_SWEEP_SPLITS=56,64,68,72,80 SLATE_C3_REPS=2 SLATE_SWEEP_OUT=gpurun_out/c3_sweep_r2.json \
  timeout 300 python tools/c3_sweep.py > gpurun_out/c3_sweep_r2.txt 2>&1
timeout 300 python tools/c3_interference.py > gpurun_out/c3_interference.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/launches_c2.csv python bench.py --steps 2 --warmup 1 --no-c3 --no-c4 --no-cpu-baseline \
  > gpurun_out/launches_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:slate_worker -c 4 \
  -o gpurun_out/prof_c2 python tools/ncu_target.py 1 > gpurun_out/prof_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:slate_worker|gemm" -c 2 \
  -o gpurun_out/prof_c3 python tools/ncu_target_c3.py 1 > gpurun_out/prof_c3.log 2>&1
ls -la gpurun_out | tail -20

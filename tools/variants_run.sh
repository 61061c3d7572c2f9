# development sweep over compile-time variants (build/variants/libslate_*.so)
for lib in build/variants/libslate_*.so; do
  v=$(basename $lib .so)
  echo "=== $v"
  export SLATE_LIB=$PWD/$lib
  [ -n "$GEMM" ] && timeout 120 python tools/gemm_check.py 2>&1 | grep -E "TFLOP|False"
  [ -n "$INTERF" ] && timeout 200 python tools/c3_interference.py 2>&1 | grep gemm
  [ -n "$SPLITS" ] && SLATE_SWEEP_SPLITS=$SPLITS SLATE_SWEEP_OUT=gpurun_out/c3_$v.json SLATE_C3_REPS=1 timeout 200 python tools/c3_sweep.py 2>&1 | tail -4
  [ -n "$NCU" ] && timeout 200 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:gemm -c 1 python tools/ncu_target_c3.py 1 2>&1 | grep -E "dram__|gpu__time"
done
true

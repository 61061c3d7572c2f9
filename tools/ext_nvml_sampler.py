import pynvml as N, time, sys
N.nvmlInit(); h = N.nvmlDeviceGetHandleByIndex(0)
t_end = time.time() + float(sys.argv[1])
while time.time() < t_end:
    N.nvmlDeviceGetClockInfo(h, N.NVML_CLOCK_SM); N.nvmlDeviceGetCurrentClocksEventReasons(h); time.sleep(0.01)

import time, traceback
try:
    import pynvml as N
    N.nvmlInit()
    h = N.nvmlDeviceGetHandleByIndex(0)
    print("max", N.nvmlDeviceGetMaxClockInfo(h, N.NVML_CLOCK_SM))
    t=time.time(); 
    for i in range(100): sm = N.nvmlDeviceGetClockInfo(h, N.NVML_CLOCK_SM)
    print("clock", sm, "per call us", (time.time()-t)/100*1e6)
    r = N.nvmlDeviceGetCurrentClocksThrottleReasons(h); print("reasons", hex(r))
    print(N.nvmlClocksThrottleReasonHwSlowdown, N.nvmlClocksThrottleReasonSwPowerCap)
except Exception:
    traceback.print_exc()

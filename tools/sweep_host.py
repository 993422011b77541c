"""Host cost of enqueueing the C5 sweep (dts_sweep_run) with the device idle,
and of the Python marshalling around it.  Needs a B200."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gc  # noqa: E402

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

insts = gen.config_instances("C5")
hs = [dts.create(i) for i in insts]
st = torch.cuda.current_stream()
o = dts.dts_run_opts_default(cuda_stream=st.cuda_stream)
for h in hs:
    dts.dts_instance_upload(h, 0, st.cuda_stream)
torch.cuda.synchronize()
gc.disable()
lib = dts.load_library()
import ctypes as C  # noqa: E402
arr = (C.c_void_p * len(hs))(*[h.handle for h in hs])
for rep in range(8):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    r = lib.dts_sweep_run(arr, len(hs), dts.DTS_POLICY_DARTS_LUF, C.byref(o), None, 0)
    t3 = time.perf_counter()
    torch.cuda.synchronize()
    print(f"python enqueue {1e3 * (t1 - t0):.2f} ms, device {1e3 * (t2 - t1):.1f} ms, "
          f"raw C call enqueue {1e3 * (t3 - t2):.2f} ms", flush=True)
# the bench's device-timed step: events around the enqueue, an L2 flush before
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device="cuda")
for rep in range(5):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    flush.zero_()
    a.record(st)
    t0 = time.perf_counter()
    dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
    t1 = time.perf_counter()
    b.record(st)
    lm = max(dts.dts_run_times(h)[0] for h in hs)
    t2 = time.perf_counter()
    print(f"step {a.elapsed_time(b):.1f} ms, loop {lm:.1f} ms, enqueue {1e3 * (t1 - t0):.2f} ms, "
          f"run_times loop {1e3 * (t2 - t1):.1f} ms", flush=True)
# the same with bench.py's nvidia-smi clock sampler running
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from bench import Clocks  # noqa: E402
with Clocks(0):
    for rep in range(5):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        flush.zero_()
        a.record(st)
        t0 = time.perf_counter()
        dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
        t1 = time.perf_counter()
        b.record(st)
        lm = max(dts.dts_run_times(h)[0] for h in hs)
        print(f"[clocks] step {a.elapsed_time(b):.1f} ms, loop {lm:.1f} ms, enqueue {1e3 * (t1 - t0):.2f} ms",
              flush=True)
# the same after fetching every result with host copies (as bench.py does after warm-up)
res0 = [dts.dts_result(h) for h in hs]
for rep in range(5):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    flush.zero_()
    a.record(st)
    t0 = time.perf_counter()
    dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
    t1 = time.perf_counter()
    b.record(st)
    lm = max(dts.dts_run_times(h)[0] for h in hs)
    print(f"[after results] step {a.elapsed_time(b):.1f} ms, loop {lm:.1f} ms, enqueue {1e3 * (t1 - t0):.2f} ms",
          flush=True)
del res0

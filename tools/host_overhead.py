"""Host-side cost of enqueueing a run (wall clock of the C-ABI calls) vs device time."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import gen
import paper_conf_ipps_gonthiermt22_b200 as dts

for name, insts in (("C1", gen.config_instances("C1")), ("C2", gen.config_instances("C2"))):
    hs = [dts.create(i) for i in insts]
    st = torch.cuda.current_stream()
    o = dts.dts_run_opts_default(cuda_stream=st.cuda_stream)
    for h in hs:
        dts.dts_instance_upload(h, 0, st.cuda_stream)
    torch.cuda.synchronize()
    for rep in range(6):
        t0 = time.perf_counter()
        dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
        t1 = time.perf_counter()
        torch.cuda.synchronize()
        t2 = time.perf_counter()
        print(f"{name} rep {rep}: enqueue {1e3*(t1-t0):.2f} ms, enqueue+run {1e3*(t2-t0):.2f} ms")
    for rep in range(3):
        t0 = time.perf_counter()
        for h in hs:
            dts.dts_run(h, dts.DTS_POLICY_DARTS_LUF, o)
        t1 = time.perf_counter()
        torch.cuda.synchronize()
        t2 = time.perf_counter()
        print(f"{name} dts_run x{len(hs)}: enqueue {1e3*(t1-t0):.2f} ms, +run {1e3*(t2-t0):.2f} ms")

"""Host cost of enqueueing the C5 sweep (wall clock of dts_sweep_run) vs its
device time.  Needs a B200."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
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
for rep in range(4):
    t0 = time.perf_counter()
    dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    print(f"C5 rep {rep}: enqueue {1e3 * (t1 - t0):.1f} ms, enqueue+run {1e3 * (t2 - t0):.1f} ms, "
          f"loop {dts.dts_run_times(hs[0])[0]:.1f} ms", flush=True)

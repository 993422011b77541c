"""Host-side phases of one end-to-end step (bench.py's e2e leg) for a workload:
uploads, sweep enqueue, device wait, batched fetch, per-instance results.
python tools/e2e_phases.py [C2|C5].  Needs a B200."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

w = sys.argv[1] if len(sys.argv) > 1 else "C2"
insts = gen.config_instances(w)
hs = [dts.create(i) for i in insts]
o = dts.dts_run_opts_default()
for h in hs:
    dts.dts_instance_upload(h, 0, None)
dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
dts.dts_fetch_results(hs)
torch.cuda.synchronize()
for rep in range(3):
    t = [time.perf_counter()]
    for h in hs:
        dts.dts_instance_upload(h, 0, None)
    t.append(time.perf_counter())
    dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
    t.append(time.perf_counter())
    torch.cuda.synchronize()
    t.append(time.perf_counter())
    dts.dts_fetch_results(hs)
    t.append(time.perf_counter())
    rs = [dts.dts_result(h) for h in hs]
    t.append(time.perf_counter())
    names = ["uploads", "sweep enqueue", "device wait", "fetch", "results (python)"]
    print(w, " ".join(f"{n}={1e3 * (t[i + 1] - t[i]):.1f}ms" for i, n in enumerate(names)),
          f"total={1e3 * (t[-1] - t[0]):.1f}ms", flush=True)

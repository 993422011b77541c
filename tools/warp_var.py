"""Same-box A/B of library variants on the one-warp path:
    python tools/warp_var.py LIB.so [LIB2.so ...]
Loop time of the longest C5 chains, C2's batch and the whole C5 sweep (median
of 3); each variant in its own process.  Needs a B200."""
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if len(sys.argv) > 2 or (len(sys.argv) == 2 and not sys.argv[1].startswith("--one=")):
    for lib in sys.argv[1:]:
        subprocess.run([sys.executable, __file__, "--one=" + lib], check=False)
    sys.exit(0)
lib = sys.argv[1][len("--one="):]
sys.path.insert(0, ROOT)
import gc  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

dts.load_library(lib)
gc.disable()
out = []
for N, M, K in ((160, 4, 1), (160, 4, 7), (100, 35, 4)):
    inst = gen.sweep_instance(N, M, K)
    out.append(f"{N},{M},{K}={statistics.median(dts.schedule(inst).loop_ms for _ in range(3)):.2f}")


def batch(insts):
    hs = [dts.create(i) for i in insts]
    o = dts.dts_run_opts_default()
    ts = []
    for _ in range(3):
        dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
        dts.dts_fetch_results(hs)
        ts.append(dts.dts_run_times(hs[0])[0])
    return statistics.median(ts)


out.append(f"C2={batch(gen.config_instances('C2')):.2f}")
out.append(f"C5={batch(gen.config_instances('C5')):.1f}")
print(os.path.basename(lib), " ".join(out), flush=True)

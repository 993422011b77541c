"""Same-box A/B of library builds: python tools/lib_ab.py LIB.so [reps].
Loop time (CUDA events around the loop kernel) of C2's critical instance,
of the whole C2 batch and of C3; median over reps.  Needs a B200."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

lib = sys.argv[1]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 7
dts.load_library(lib)
import gen  # noqa: E402

c2 = gen.config_instances("C2")
one = dts.create(c2[19])
o = dts.dts_run_opts_default()
t1 = []
for _ in range(reps):
    dts.dts_run(one, dts.DTS_POLICY_DARTS_LUF, o)
    t1.append(dts.dts_result(one).loop_ms)
hs = [dts.create(i) for i in c2]
tb = []
for _ in range(reps):
    dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
    tb.append(max(dts.dts_result(h).loop_ms for h in hs))
c3 = dts.create(gen.config_instances("C3")[0])
t3 = []
for _ in range(3):
    dts.dts_run(c3, dts.DTS_POLICY_DARTS_LUF, o)
    t3.append(dts.dts_result(c3).loop_ms)
print(f"{os.path.basename(lib):24s} C2[19] {statistics.median(t1):.3f} ms  C2 batch {statistics.median(tb):.3f} ms  "
      f"C3 {statistics.median(t3):.2f} ms", flush=True)

"""Print the per-phase cycle split of the decision loop (dts_result_view.prof_cycles)
for a few instances, plus loop time per decision.  Needs a B200."""
import os
os.environ.setdefault("DTS_PROFILE", "1")
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

NAMES = ["pop", "argmax", "plan", "serve_loads", "luf", "evict", "seg_load", "other"]
cases = [gen.matmul2d(100, M=35, K=4), gen.matmul3d(40, M=142, K=4)]
blocks = (0, 64, 256)
if len(sys.argv) > 1 and sys.argv[1] == "big":
    cases = [gen.config_instances("C4a")[0], gen.config_instances("C4b")[0]]
    blocks = (0,)
for inst in cases:
    for block in blocks:
        for smem in (0,):
            dts.schedule(inst, block_threads=block, smem_budget=smem)
            g = dts.schedule(inst, block_threads=block, smem_budget=smem)
            tot = sum(g.prof_cycles[:4]) + g.prof_cycles[7]
            print(f"{inst.name} block={block} smem={smem}: loop {g.loop_ms:.2f} ms, "
                  f"{g.n_served} dec, {g.n_scans} scans ({g.n_fallback2} fb2, {g.n_fallback_first} fbf), {g.n_loads} loads, "
                  f"{1e6 * g.loop_ms / max(g.n_served, 1):.0f} ns/dec, total_ms {g.total_ms:.2f}")
            print("   cycles/scan: " + ", ".join(
                f"{n}={c / max(g.n_scans, 1):.0f}" for n, c in zip(NAMES, g.prof_cycles)))
            print(f"   pop cycles/pop: {g.prof_cycles[0] / max(g.n_served - g.n_scans, 1):.0f}; "
                  f"batches {g.prof_cycles[10]} ({g.prof_cycles[11]} pops): warp0 "
                  f"{g.prof_cycles[8] / max(g.prof_cycles[10], 1):.0f} cyc, rank phase "
                  f"{g.prof_cycles[9] / max(g.prof_cycles[10], 1):.0f} cyc per batch; w0 checkpoints "
                  + " ".join(f"{g.prof_cycles[i] / max(g.prof_cycles[10], 1):.0f}" for i in range(12, 16)))

"""Mutation check of the CPU oracle's pins (test infrastructure).

Each mutant is a plausible mistake in oracle/dts_oracle.c (a dropped key, a
wrong credit, a swapped order, a missing rule).  The mutant is compiled to a
scratch library and the CPU pin suite (tests/test_oracle_pins.py) is run
against it through DTS_ORACLE_LIB.  A mutant is KILLED when at least one pin
fails.  A mutant listed as `equivalent` cannot be killed: its change is
unreachable under the model (the reason is given; DESIGN.md restates it).

usage: python tests/oracle_mutants.py [--out profiles/r02_oracle_mutants.txt]
"""
import argparse
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "dts_oracle.c")

# (name, old, new, expected) -- `old` must occur exactly once
MUTANTS = [
    ("3inputs key drops u(D) (R24)",
     "better(s->cnt_n2[D], s->cnt_u[D], D, s->cnt_n2[b2], s->cnt_u[b2], b2)",
     "better(s->cnt_n2[D], 0, D, s->cnt_n2[b2], 0, b2)", "killed"),
    ("3inputs key ordered (u, n2) instead of (n2, u)",
     "better(s->cnt_n2[D], s->cnt_u[D], D, s->cnt_n2[b2], s->cnt_u[b2], b2)",
     "better(s->cnt_u[D], s->cnt_n2[D], D, s->cnt_u[b2], s->cnt_n2[b2], b2)", "killed"),
    ("n2 credits only the first (lower-id) missing input (R6)",
     "s->cnt_n2[miss[0]]++; s->cnt_n2[miss[1]]++;",
     "s->cnt_n2[miss[0]]++;", "killed"),
    ("n2 credits only the second missing input",
     "s->cnt_n2[miss[0]]++; s->cnt_n2[miss[1]]++;",
     "s->cnt_n2[miss[1]]++;", "killed"),
    ("3inputs task: any available task using D2 (ignores its missing count)",
     "if (s->avail[T] && uses(s, T, b2) && missing(s, k, T) == 2) {",
     "if (s->avail[T] && uses(s, T, b2)) {", "killed"),
    ("3inputs task: lowest-id available task (ignores D2)",
     "if (s->avail[T] && uses(s, T, b2) && missing(s, k, T) == 2) {",
     "if (s->avail[T]) {", "killed"),
    ("main key drops u(D) (R23)",
     "better(s->cnt_n[D], s->cnt_u[D], D, s->cnt_n[best], s->cnt_u[best], best)",
     "better(s->cnt_n[D], 0, D, s->cnt_n[best], 0, best)", "killed"),
    ("main key ordered (u, n) instead of (n, u)",
     "better(s->cnt_n[D], s->cnt_u[D], D, s->cnt_n[best], s->cnt_u[best], best)",
     "better(s->cnt_u[D], s->cnt_n[D], D, s->cnt_u[best], s->cnt_n[best], best)", "killed"),
    ("u(D) also counts allocated tasks (R2)",
     "        if (!s->avail[T]) continue;\n        int32_t miss[2] = {-1, -1};",
     "        if (!s->avail[T]) { for (int64_t e2 = s->dp[T]; e2 < s->dp[T + 1]; e2++) s->cnt_u[s->dd[e2]]++; continue; }\n        int32_t miss[2] = {-1, -1};",
     "killed"),
    ("LUF ignores np (lowest id with nb = 0)",
     "if (V < 0 || np < Vnp) { V = D; Vnp = np; }",
     "if (V < 0) { V = D; Vnp = np; }", "killed"),
    ("LUF ties to the highest id",
     "if (V < 0 || np < Vnp) { V = D; Vnp = np; }",
     "if (V < 0 || np <= Vnp) { V = D; Vnp = np; }", "killed"),
    ("LUF takes the MOST used datum",
     "if (V < 0 || np < Vnp) { V = D; Vnp = np; }",
     "if (V < 0 || np > Vnp) { V = D; Vnp = np; }", "killed"),
    ("Alg. 6 l.8 dropped: planned tasks keep an evicted input",
     "if (uses(s, T, V)) { s->avail[T] = 1; returned = 1; }",
     "if (0) { s->avail[T] = 1; returned = 1; }", "killed"),
    ("bus not FIFO: a load starts at its request time",
     "int64_t st = s->bus_free > t ? s->bus_free : t;",
     "int64_t st = t;", "killed"),
    ("transfer time rounded down instead of up (R9)",
     "* 1000000000u + (s->bw - 1);",
     "* 1000000000u;", "killed"),
    ("W=0 asks for the next task at the start of the current one (R7)",
     "if (s->W == 0) s->req[k] = end;",
     "if (s->W == 0) s->req[k] = start;", "killed"),
    ("OPTI takes the best datum instead of the first (R28)",
     "            best = D;\n            break;",
     "            if (best < 0 || better(s->cnt_n[D], s->cnt_u[D], D, s->cnt_n[best], s->cnt_u[best], best)) best = D;\n            continue;",
     "killed"),
    ("Belady counts the running task's use as a next use (R29)",
     "const int started = i < nbuf - 1 && s->r->task_start[Tb] <= s->now;",
     "const int started = 0;", "killed"),
    ("Belady eviction takes effect at the request, not when the running task ends",
     "const int64_t te = s->evict_at > t ? s->evict_at : t;",
     "const int64_t te = t;", "killed"),
    ("Belady ties to the highest id",
     "if (pos > far) { far = pos; V = D; }",
     "if (pos >= far) { far = pos; V = D; }", "killed"),
    ("W >= 2 asks when its last task starts (as W = 1)",
     "else if (s->n_on[k] < s->W) s->req[k] = t;",
     "else if (1) s->req[k] = r->task_start[T];", "killed"),
    ("R18 removed: idle GPUs are not woken when planned tasks return",
     "if (s->idle[j]) { s->idle[j] = 0; s->req[j] = t; s->r->n_wakes++; }",
     "if (0) { s->idle[j] = 0; s->req[j] = t; s->r->n_wakes++; }",
     "equivalent: a return comes from the plan made at the same request out of a non-empty "
     "pool, while an idle GPU saw an empty pool, and the pool only refills by returns -- so no "
     "GPU is idle when a return happens (DESIGN.md, reading R18; the oracle counts wakes)"),
]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    src = open(SRC).read()
    lines = []
    bad = 0
    with tempfile.TemporaryDirectory() as tmp:
        for i, (name, old, new, expect) in enumerate(MUTANTS):
            assert src.count(old) == 1, f"mutant {name!r}: pattern occurs {src.count(old)} times"
            c = os.path.join(tmp, f"m{i}.c")
            so = os.path.join(tmp, f"m{i}.so")
            open(c, "w").write(src.replace(old, new))
            subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", so, c])
            env = dict(os.environ, DTS_ORACLE_LIB=so)
            p = subprocess.run([sys.executable, "-m", "pytest", "-q", "-p", "no:cacheprovider",
                                os.path.join(ROOT, "tests", "test_oracle_pins.py")],
                               env=env, cwd=ROOT, capture_output=True, text=True)
            tail = [ln for ln in p.stdout.splitlines() if ln.strip()][-1:]
            killed = p.returncode != 0
            status = "KILLED" if killed else "survived"
            ok = killed == expect.startswith("killed")
            bad += not ok
            lines.append(f"{status:8s} {'ok ' if ok else 'BAD'} {name}: {tail[0] if tail else ''}"
                         + ("" if expect == "killed" else f"\n         expected {expect}"))
            print(lines[-1], flush=True)
    txt = "\n".join(lines) + f"\n{len(MUTANTS)} mutants, {bad} not as expected\n"
    if args.out:
        open(os.path.join(ROOT, args.out), "w").write(txt)
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())

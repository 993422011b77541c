# same-box A/B: luf_victim on warp 0 alone for short resident lists (LUF_WARP_MAX), then checks
O=gpurun_out
for r in 1 2; do
for L in tools/var/v_base.so tools/var/v_lufw.so tools/var/v_lufw32.so; do
  timeout 300 python tools/lib_ab.py $L 9 2>&1 | tail -1
done; done | tee $O/r01o_lib_ab_lufwarp.txt
timeout 1500 python -m pytest tests -m gpu -x -q > $O/r01o_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/r01o_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > $O/r01o_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/r01o_smoke.log
timeout 300 python tools/san_c5.py 6 > $O/r01o_rep.log 2>&1; echo "C5 rep x6 rc=$?"; tail -1 $O/r01o_rep.log
DTS_BLOCK=128 timeout 900 compute-sanitizer --tool synccheck --print-limit 10 python tools/san_c5.py 1 16 > $O/r01o_sync.log 2>&1; echo "synccheck rc=$?"; grep -v "^=========     " $O/r01o_sync.log | tail -2
timeout 600 python bench.py > $O/r01o_bench_C2.json 2> $O/r01o_bench_C2.err; echo "C2 rc=$?"; cat $O/r01o_bench_C2.json
timeout 900 python bench.py --workload C5 --steps 5 > $O/r01o_bench_C5.json 2> $O/r01o_bench_C5.err; echo "C5 rc=$?"

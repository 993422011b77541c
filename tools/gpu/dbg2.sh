O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
DTS_POISON=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > $O/dbg2_pytest.log 2>&1; echo "poison pytest rc=$?"; tail -30 $O/dbg2_pytest.log | grep -v "^\s*$" | tail -25
for B in 128 64; do DTS_POISON=1 DTS_BLOCK=$B timeout 300 python tools/san_c5.py 3 > $O/dbg2_rep_$B.log 2>&1; echo "poison rep block $B rc=$?"; tail -2 $O/dbg2_rep_$B.log; done
DTS_POISON=1 DTS_BLOCK=128 timeout 900 compute-sanitizer --tool memcheck --print-limit 10 python tools/san_c5.py 1 > $O/dbg2_san.log 2>&1; echo "san rc=$?"; grep -v "^=========     " $O/dbg2_san.log | head -40

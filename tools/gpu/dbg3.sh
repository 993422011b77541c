O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
DTS_BLOCK=128 timeout 300 python tools/san_c5.py 20 > $O/dbg3_rep.log 2>&1; echo "rep128 x20 rc=$?"; tail -2 $O/dbg3_rep.log
DTS_BLOCK=128 timeout 1200 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 20 python tools/san_c5.py 1 16 > $O/dbg3_race.log 2>&1; echo "race rc=$?"; grep -v "^=========     " $O/dbg3_race.log | head -40
DTS_BLOCK=128 timeout 600 compute-sanitizer --tool synccheck --print-limit 20 python tools/san_c5.py 1 16 > $O/dbg3_sync.log 2>&1; echo "sync rc=$?"; grep -v "^=========     " $O/dbg3_sync.log | head -20
DTS_BLOCK=128 timeout 1500 compute-sanitizer --tool memcheck --print-limit 10 python tools/san_c5.py 12 > $O/dbg3_mem.log 2>&1; echo "mem rc=$?"; grep -v "^=========     " $O/dbg3_mem.log | head -60

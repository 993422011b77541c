O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for r in 1 2; do
for L in tools/oldlib_75692b6.so tools/oldlib_1d7b8ac.so tools/oldlib_0b842ed.so paper_conf_ipps_gonthiermt22_b200/lib/libdts.so; do
  timeout 300 python tools/lib_ab.py $L 9 2>&1 | tail -1
done; done

O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 300 python tools/e2e_phases.py C2
timeout 600 python tools/e2e_phases.py C5

python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python tools/prof_fine.py
timeout 300 python tools/prof_phases.py big 2>&1 | grep -v "^ *pop cycles"
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py -x -q 2>&1 | tail -3

python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python tools/prof_shard.py 2>&1 | tee gpurun_out/prof_shard.txt
timeout 600 python -m pytest tests/test_gpu_shard.py -x -q > gpurun_out/shard.log 2>&1; echo "shard rc=$?"; tail -3 gpurun_out/shard.log

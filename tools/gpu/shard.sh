set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_shard.py -x -q -k "not ipc and not full_digest" > gpurun_out/shard.log 2>&1; echo "shard rc=$?"
tail -30 gpurun_out/shard.log
timeout 300 python -m pytest tests/test_gpu_shard.py -x -q -k "ipc" > gpurun_out/shard_ipc.log 2>&1; echo "ipc rc=$?"
tail -30 gpurun_out/shard_ipc.log
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/parity.log 2>&1; echo "parity rc=$?"
tail -3 gpurun_out/parity.log

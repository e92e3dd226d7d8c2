mkdir -p gpurun_out
python __graft_entry__.py
timeout 1800 python -m pytest tests -m gpu -q --durations=8 > gpurun_out/tests.log 2>&1
tail -30 gpurun_out/tests.log

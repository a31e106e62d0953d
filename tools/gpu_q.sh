mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_p2p.py -q -x -m gpu --durations=5 -k "repeated or large or unsupported or ipc" 2>&1 | tail -15

python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/dbg_p2p.py 1 2 3 2>&1 | tail -6
timeout 900 python -m pytest tests/test_gpu_p2p.py -q -x -m gpu --durations=4 2>&1 | tail -8
timeout 300 python bench.py --force-dist --steps 3 --warmup 3 --no-engines --no-cpu 2>&1 | tail -1 | cut -c1-300

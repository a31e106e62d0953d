mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02i_build.log 2>&1 || tail -20 gpurun_out/r02i_build.log
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "small_cluster or rows_and_pma or integer" 2>&1 | tail -3
timeout 120 python tools/quickbench.py --configs heat2d-256 --engines rdg_cuda --fuse 0 --T 10 2>&1 | cut -c1-110
timeout 120 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:small2d python tools/prof_step.py --workload heat2d-256 --engine auto --fuse 0 --T 10 2>&1 | grep -E "duration" | head -3
timeout 1500 python -m pytest tests -m gpu -q --durations=3 -rf > gpurun_out/r02i_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02i_pytest_gpu.log
tail -8 gpurun_out/r02i_pytest_gpu.log

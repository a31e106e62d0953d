mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02e_build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x --durations=8 -rf > gpurun_out/r02e_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02e_pytest_gpu.log
tail -25 gpurun_out/r02e_pytest_gpu.log
timeout 600 python tools/quickbench.py --configs heat2d-256,box2d9p-10240,box2d49p-10240,heat3d-512,box3d27p-512 --engines auto --fuse 0 --T 100 2>&1 | tee gpurun_out/r02e_quickbench.jsonl | cut -c1-160

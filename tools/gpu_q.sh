mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "rows_and_pma or 2d_parity_small or fusion or integer" 2>&1 | tail -3
for pma in 0 1; do LORA_RDG_PMA=$pma timeout 300 python tools/quickbench.py --configs box2d49p-10240 --engines rdg_cuda --fuse 1,2 --T 40; done
timeout 300 python tools/quickbench.py --configs box2d49p-10240 --engines rdg_cuda --fuse 1 --T 100

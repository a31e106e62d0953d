timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_p2p.py -q -x -k "3d" 2>&1 | tail -2
bash tools/gpu_variants.sh r02m box3d27p-512,heat3d-512 2,3 lag0 2>&1 | tail -12

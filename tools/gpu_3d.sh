for v in w16 w12; do LORA_LIB=variants_tmp/$v.so timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "3d" 2>&1 | tail -1; done
bash tools/gpu_variants.sh r02q box3d27p-512,heat3d-512 2 w16 w12 2>&1 | tail -8

python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "small_cluster" 2>&1 | tail -1
for v in base t1024 t256; do for rp in 1 2 4; do
  LIB=paper_conf_sc_zhanglyczcy24_b200/liblora_stencil.so; [ $v != base ] && LIB=variants_tmp/$v.so
  echo "== $v rp=$rp $(LORA_SMALL_RP=$rp LORA_LIB=$LIB timeout 120 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:small2d python tools/quickbench.py --configs heat2d-256 --engines rdg_cuda --fuse 0 --T 10 2>&1 | grep -E "duration" | tail -1 | tr -s ' ')"
done; done

python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "small_cluster" 2>&1 | tail -2
for v in base b1 b2 b8; do
  LIB=paper_conf_sc_zhanglyczcy24_b200/liblora_stencil.so; [ $v != base ] && LIB=variants_tmp/$v.so
  echo "== $v"; LORA_LIB=$LIB timeout 120 python tools/quickbench.py --configs heat2d-256 --engines rdg_cuda --fuse 0 --T 10 2>&1 | cut -c1-110
done
timeout 120 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none -k regex:small2d python tools/prof_step.py --workload heat2d-256 --engine auto --fuse 0 --T 10 2>&1 | grep -E "duration|inst_exec" | head -3

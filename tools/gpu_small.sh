python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "small_cluster" 2>&1 | tail -2
for m in "LORA_SMALL_RP=2" "LORA_SMALL_RP=4" "LORA_SMALL_RP=8"; do
  echo "== $m"; env $m timeout 120 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:small2d python tools/prof_step.py --workload heat2d-256 --engine auto --fuse 0 --T 10 2>&1 | grep -E "duration" | head -3
  env $m timeout 120 python tools/quickbench.py --configs heat2d-256 --engines rdg_cuda --fuse 0 --T 10 2>&1 | cut -c1-100
done

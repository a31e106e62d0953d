mkdir -p gpurun_out
for v in base b1 b2 b4; do
  LIB=paper_conf_sc_zhanglyczcy24_b200/liblora_stencil.so; [ $v != base ] && LIB=variants_tmp/$v.so
  echo "== $v"; LORA_LIB=$LIB timeout 120 python tools/quickbench.py --configs heat2d-256 --engines rdg_cuda --fuse 0 --T 10 2>&1 | cut -c1-110
done
timeout 300 ncu --metrics gpu__time_duration.sum,sm__cycles_elapsed.avg,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum --clock-control none -k regex:small2d python tools/prof_step.py --workload heat2d-256 --engine auto --fuse 0 --T 10 2>&1 | grep -E "small2d|duration|cycles|wavefronts" | head -12
OUT=gpurun_out/r02h_heat2d; timeout 300 ncu --set full --clock-control none --import-source on -k regex:small2d -s 2 -c 1 -o $OUT -f python tools/prof_step.py --workload heat2d-256 --engine auto --fuse 0 --T 10 > /dev/null 2>&1
python tools/ncu_summary.py $OUT.ncu-rep > $OUT.summary.json 2>/dev/null; ncu -i $OUT.ncu-rep --page source --csv > $OUT.source.csv 2>/dev/null

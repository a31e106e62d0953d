mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02f_build.log 2>&1
timeout 300 python tools/dbg_p2p3d.py 2>&1 | tail -16
timeout 1500 python -m pytest tests -m gpu -q -x --durations=8 -rf > gpurun_out/r02f_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02f_pytest_gpu.log
tail -15 gpurun_out/r02f_pytest_gpu.log
bash tools/gpu_variants.sh r02f box2d49p-10240 2 nh1 pf0 u1 rc256 2>&1 | tail -8
OUT=gpurun_out/r02f_box2d49p-10240_auto_k0
timeout 600 ncu --set full --clock-control none --import-source on -k regex:rdg2d_kernel -s 3 -c 1 -o $OUT -f python tools/prof_step.py --workload box2d49p-10240 --engine auto --fuse 0 --T 16 > $OUT.log 2>&1
ncu -i $OUT.ncu-rep --page raw --csv > $OUT.raw.csv 2>/dev/null; python tools/ncu_summary.py $OUT.ncu-rep > $OUT.summary.json 2>/dev/null
ncu -i $OUT.ncu-rep --page source --csv > $OUT.source.csv 2>/dev/null

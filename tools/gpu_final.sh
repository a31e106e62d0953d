#!/bin/bash
# Full measurement call: build, GPU tests, smoke, bench (+ reference arm), ncu launch list of the bench
# command, ncu --set full of the two dominant kernels.  usage: tools/gpu_final.sh TAG
TAG=${1:-r02z}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { tail -30 gpurun_out/${TAG}_build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q --durations=8 -rf > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
tail -14 gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
tail -4 gpurun_out/${TAG}_smoke.log
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${TAG}_bench_ref.json 2> gpurun_out/${TAG}_bench_ref.err; echo "ref rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_ncu_launches.csv \
   python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --no-engines --no-configs > /dev/null 2>&1; echo "ncu launches rc=$?"
for spec in "rdg2d_kernel:box2d49p-10240" "rdg3df_kernel:box3d27p-512"; do
  IFS=: read -r KRE WL <<< "$spec"
  OUT=gpurun_out/${TAG}_${WL}
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KRE} -s 3 -c 1 -o $OUT -f \
     python tools/prof_step.py --workload $WL --engine auto --fuse 0 --T 16 > $OUT.log 2>&1; echo "ncu $spec rc=$?"
  python tools/ncu_summary.py $OUT.ncu-rep > $OUT.summary.json 2>/dev/null
done
python - <<PY
import json
d=json.loads(open("gpurun_out/${TAG}_bench.json").read())
print('main', round(d['value'],1), d['roofline']['bound'], round(d['roofline']['frac'],3), 'e2e', round(d['e2e']['value'],1), d['clocks'])
for k,v in d['configs'].items(): print(k, round(v['value'],1), v['fuse_k'], v['roofline']['bound'], round(v['roofline']['frac'],3), v['clocks'].get('sm_mhz'), v['clocks']['reasons'])
for k,v in d['engines'].items(): print(k, round(v.get('GStencil_s',0),1), v.get('fuse_k'))
print('cpu', d['cpu_baseline'])
PY
cut -c1-400 gpurun_out/${TAG}_bench_ref.json

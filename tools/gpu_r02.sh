#!/bin/bash
# Round-2 GPU call: build, FP64 peak, variants quickbench, gpu tests, smoke, bench, ncu launch list.
TAG=${1:-r02a}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
timeout 300 python tools/fp64_peak.py ${TAG} > gpurun_out/${TAG}_fp64_peak.log 2>&1; echo "fp64 rc=$?"
cp profiles/${TAG}_fp64_peak.json gpurun_out/ 2>/dev/null
if ls variants_tmp/*.so >/dev/null 2>&1; then
  bash tools/gpu_variants.sh ${TAG} ${VCFG:-box2d49p-10240} ${VFUSE:-2} $(cd variants_tmp && ls *.so | sed 's/\.so$//') 2>&1 | tail -20
fi
timeout 2400 python -m pytest tests -m gpu -q --durations=15 -rf > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
tail -25 gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
tail -4 gpurun_out/${TAG}_smoke.log
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"
cut -c1-1500 gpurun_out/${TAG}_bench.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
   python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --no-engines --no-configs > /dev/null 2>&1; echo "ncu launches rc=$?"

#!/bin/bash
# One GPU call: build, gpu tests, smoke, bench (+per-stencil), ncu launch list of the bench, ncu --set full captures.
# usage: tools/gpu_round.sh TAG "kregex:workload:engine:fuse" ...
TAG=${1:-r01}; shift
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
tail -3 gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
tail -4 gpurun_out/${TAG}_smoke.log
timeout 900 python bench.py --per-stencil > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"
cat gpurun_out/${TAG}_bench.json
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${TAG}_bench_ref.json 2>&1; echo "ref rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
   python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --no-engines > /dev/null 2>&1; echo "ncu launches rc=$?"
for spec in "$@"; do
  IFS=: read -r KRE WL ENG FK <<< "$spec"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KRE} -s 3 -c 1 \
     -o gpurun_out/${TAG}_${WL}_${ENG}_k${FK} -f python tools/prof_step.py --workload $WL --engine $ENG --fuse $FK --T 16 > gpurun_out/${TAG}_${WL}_${ENG}_k${FK}.log 2>&1
  echo "ncu $spec rc=$?"
done

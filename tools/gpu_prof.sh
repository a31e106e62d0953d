#!/bin/bash
# GPU call: build, selected tests, quickbench, ncu --set full captures with source pages.
# usage: TESTS="pytest args" QB="configs" tools/gpu_prof.sh TAG "kregex:workload:engine:fuse" ...
TAG=$1; shift
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { tail -30 gpurun_out/${TAG}_build.log; exit 1; }
if [ -n "$TESTS" ]; then
  timeout 1200 python -m pytest $TESTS -q -x -rf > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest.log
  tail -15 gpurun_out/${TAG}_pytest.log
fi
if [ -n "$QB" ]; then
  timeout 600 python tools/quickbench.py --configs $QB --engines ${QBE:-auto} --fuse ${QBF:-0} --T ${QBT:-40} 2>&1 | tee gpurun_out/${TAG}_quickbench.jsonl | cut -c1-200
fi
if [ -n "$VARIANTS" ]; then
  bash tools/gpu_variants.sh ${TAG} ${VCFG:-box2d49p-10240} ${VFUSE:-2} $VARIANTS 2>&1 | tail -20
fi
for spec in "$@"; do
  IFS=: read -r KRE WL ENG FK <<< "$spec"
  OUT=gpurun_out/${TAG}_${WL}_${ENG}_k${FK}
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KRE} -s 3 -c 1 \
     -o $OUT -f python tools/prof_step.py --workload $WL --engine $ENG --fuse $FK --T 16 > $OUT.log 2>&1
  echo "ncu $spec rc=$?"
  ncu -i $OUT.ncu-rep --page source --csv > $OUT.source.csv 2>/dev/null
  ncu -i $OUT.ncu-rep --page raw --csv > $OUT.raw.csv 2>/dev/null
  python tools/ncu_summary.py $OUT.ncu-rep > $OUT.summary.json 2>/dev/null
done

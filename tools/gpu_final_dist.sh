#!/bin/bash
TAG=$1
bash tools/gpu_final.sh $TAG   # then one-rank runs through the P2P exchange path on the multi-GPU slabs
for wl in box2d49p-40960 box3d27p-1024; do
  timeout 900 python bench.py --force-dist --workload $wl --no-e2e --no-cpu --no-engines --no-configs --steps 3 --warmup 3 > gpurun_out/${TAG}_forcedist_$wl.json 2> gpurun_out/${TAG}_forcedist_$wl.err
  python -c "import json; d=json.load(open('gpurun_out/${TAG}_forcedist_$wl.json')); print('$wl', d['value'], d['config']['exchange'][:20], d['clocks'])"
done

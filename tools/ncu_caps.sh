#!/bin/bash
# usage: tools/ncu_caps.sh TAG "kregex:workload:engine:fuse" ...
TAG=$1; shift
python paper_conf_sc_zhanglyczcy24_b200/_build.py > /dev/null
for spec in "$@"; do
  IFS=: read -r KRE WL ENG FK <<< "$spec"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KRE} -s 3 -c 1 \
     -o gpurun_out/${TAG}_${WL}_${ENG}_k${FK} -f python tools/prof_step.py --workload $WL --engine $ENG --fuse $FK --T 16 > gpurun_out/${TAG}_${WL}_${ENG}_k${FK}.log 2>&1
  echo "ncu $spec rc=$?"
done

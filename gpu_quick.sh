#!/bin/bash
# quick GPU check: build, run gpu tests
set -x
python paper_conf_sc_zhanglyczcy24_b200/_build.py > /dev/null
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -30

#!/bin/bash
# per-phase clocks of the large-net kernels (timing build in tbuild/), then the A/B bench
FGR_FLOW_MAX=100000 FGR_LIB_PATH=tbuild/libfastgr.so timeout 300 python tools/prof_step.py t9 2>&1 | grep -E "^FLOW" | sort -t= -k2 -n | tail -12
TAG=${1:-ab}; shift
bash tools/ab_run.sh $TAG "$@"

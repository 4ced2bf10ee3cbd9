#!/bin/bash
# One ncu --set full capture of the first launch of kernel regex K in a bench run, with
# text summaries in gpurun_out/.  Usage: bash tools/prof_kern.sh TAG KREGEX [bench args...]
export PATH=/usr/local/cuda/bin:$PATH
TAG=$1; K=$2; shift 2
P=/tmp/prof; mkdir -p $P gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -f -k regex:$K -c 1 -o $P/$TAG \
  python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > gpurun_out/ncu_$TAG.log 2>&1
python tools/ncu_hot.py $P/$TAG.ncu-rep 30 > gpurun_out/$TAG.hot.txt 2>&1
python tools/ncu_mix.py $P/$TAG.ncu-rep 25 > gpurun_out/$TAG.mix.txt 2>&1
ncu -i $P/$TAG.ncu-rep --page details > gpurun_out/$TAG.details.txt 2>&1
